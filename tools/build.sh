#!/bin/bash
# Rebuild libmp.so (fails loudly) from anywhere.
cd "$(dirname "$0")/.." && python paper_conf_ipps_tayebbfg24_b200/build.py > /tmp/mpbuild.log 2>&1 || { grep -E "error" /tmp/mpbuild.log | head -20; exit 1; }
grep -E "warning" /tmp/mpbuild.log | head -5
ls -la --time-style=+%T paper_conf_ipps_tayebbfg24_b200/libmp.so
