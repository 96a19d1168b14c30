for i in 1 2; do
timeout 600 python tools/scenarios.py C3 --opts '{"_v":"new"}'
WCSVD_LIBRARY=tools/exp/lib_fww.so timeout 600 python tools/scenarios.py C3 --opts '{"_v":"flat_with_wcycle"}'
WCSVD_PKG_DIR=tools/exp/headpkg timeout 600 python tools/scenarios.py C3 --opts '{"_v":"head"}'
done
