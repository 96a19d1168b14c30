for i in 1 2; do
timeout 600 python tools/scenarios.py C3 "C5/4:0" 2>&1 | cut -c1-130
WCSVD_L1_NW=4 timeout 600 python tools/scenarios.py C3 "C5/4:0" 2>&1 | cut -c1-130
WCSVD_L1_NW=8 timeout 600 python tools/scenarios.py C4 2>&1 | cut -c1-130
done
