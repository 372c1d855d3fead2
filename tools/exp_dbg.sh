# debug-flag matrix of the quad kernel on 300 units of C2 (1 skip producers, 2 skip scoring, 4 skip MMA)
for dbg in 0 1 2 3 4 5 6 7; do timeout 120 python tools/run_search.py --units 300 --debug $dbg 2>&1 | tail -1 | cut -c1-80; done
