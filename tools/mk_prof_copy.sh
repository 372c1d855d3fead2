#!/bin/bash
# Instrumented copy of the repo under scratch/prof (EPI4_PROF=1 build: per-role cycle counters, debug-64 trace)
set -e
cd "$(dirname "$0")/.."
rm -rf scratch/prof && mkdir -p scratch/prof
cp -r datagen include oracle paper_conf_icpp_nobreiss22_b200 tools scratch/prof/
rm -f scratch/prof/paper_conf_icpp_nobreiss22_b200/libepi4.so
EPI4_PROF=1 python scratch/prof/paper_conf_icpp_nobreiss22_b200/build.py --force > /dev/null
echo scratch/prof built
