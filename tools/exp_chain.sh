# TMA -> MMA chain isolation on the first 300 C2 units (debug bits: 1 producers off, 2 scoring off, 4 MMA off,
# 32 MMA ignores the relay, 128 no A copies)
for dbg in 3 35 131 163 7 135 0 32; do timeout 120 python tools/run_search.py --units 300 --debug $dbg 2>&1 | tail -1 | cut -c1-110; done
