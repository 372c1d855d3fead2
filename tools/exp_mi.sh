cd variants/mi1
timeout 600 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
for r in 1 2; do
for st in 53 44; do EPI4_STAGES=$st EPI4_VERBOSE=1 timeout 120 python tools/run_search.py --units 300 2>&1 | tail -2 | sed 's/best.*quad/quad/' | cut -c1-110; done
(cd ../.. && timeout 120 python tools/run_search.py --units 300 2>&1 | tail -1 | sed 's/best.*quad/tree quad/' | cut -c1-60)
done
