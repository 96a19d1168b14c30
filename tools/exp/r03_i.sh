for pad in 0 25000 60000 0; do echo pad $pad; WCSVD_TP_SMEM_PAD=$pad timeout 300 python tools/scenarios.py C2 2>&1 | cut -c1-100; done
WCSVD_LIBRARY=tools/exp/lib_phase.so timeout 300 python tools/exp/phase_tp.py C2 10000 2>&1 | tail -12
