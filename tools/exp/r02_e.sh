for i in 1 2; do
timeout 600 python tools/scenarios.py C3 --opts '{"_v":"new"}'
WCSVD_SLOTS_ALL=1 timeout 600 python tools/scenarios.py C3 --opts '{"_v":"slots_all"}'
WCSVD_LIBRARY=tools/exp/lib_stage_old.so timeout 600 python tools/scenarios.py C3 --opts '{"_v":"stage_old"}'
WCSVD_PKG_DIR=tools/exp/headpkg timeout 600 python tools/scenarios.py C3 --opts '{"_v":"head"}'
done
