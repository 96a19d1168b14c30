set -x
mkdir -p gpurun_out
./tools/evd_probe > gpurun_out/evd_probe3.json 2>&1; cat gpurun_out/evd_probe3.json
timeout 300 python tools/exp/dump.py /tmp/new.npz
timeout 300 bash tools/exp/swap_run.sh tools/exp/libwcsvd_head.so python tools/exp/dump.py /tmp/head.npz
python tools/exp/bitcmp.py /tmp/new.npz /tmp/head.npz
for c in C3 C4 C5; do
  timeout 300 python tools/quick_time.py $c 2>&1 | tail -1
  timeout 300 bash tools/exp/swap_run.sh tools/exp/libwcsvd_head.so python tools/quick_time.py $c 2>&1 | tail -1
done
