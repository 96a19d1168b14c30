WCSVD_LIBRARY=tools/exp/lib_phase.so timeout 300 python tools/exp/phase.py C3 592 | tail -3
WCSVD_LIBRARY=tools/exp/lib_phase.so timeout 300 python tools/exp/phase.py C4 592 | tail -3
