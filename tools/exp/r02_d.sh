for i in 1 2; do
WCSVD_PKG_DIR=tools/exp/headpkg timeout 600 python tools/scenarios.py C3 --opts '{"_v":"head"}'
timeout 600 python tools/scenarios.py C3 --opts '{"_v":"new"}'
done
WCSVD_PKG_DIR=tools/exp/headpkg timeout 600 python tools/scenarios.py C5 --opts '{"_v":"head"}'
timeout 600 python tools/scenarios.py C5 "C5/8:0" "C5/4:0" --opts '{"_v":"new"}'
