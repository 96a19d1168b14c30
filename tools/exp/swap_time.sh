#!/bin/bash
# A/B timing: run quick_time with an alternative libwcsvd.so (experiments only)
set -e
ALT=$1; shift
cp paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so /tmp/libwcsvd_main.so
cp "$ALT" paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so
python tools/quick_time.py "$@" || true
cp /tmp/libwcsvd_main.so paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so
