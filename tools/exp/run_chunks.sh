timeout 600 python tools/exp/host_chunks.py C2
timeout 600 python tools/exp/host_chunks.py C4
