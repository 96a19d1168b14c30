timeout 600 python tools/exp/host_chunks.py C2 8,12,16,20,24,32
timeout 600 python tools/exp/host_chunks.py C3 4,6,8,12
