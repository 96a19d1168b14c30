#!/bin/bash
# Run an arbitrary command with an alternative libwcsvd.so in place (experiments only).
ALT=$1; shift
cp paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so /tmp/libwcsvd_main.so
cp "$ALT" paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so
"$@"
cp /tmp/libwcsvd_main.so paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so
