for r in 1 2; do
  for g in 148 146 144 140; do timeout 120 python tools/run_search.py --grid $g 2>&1 | tail -1 | sed "s/best.*quad \([0-9.]*\) ms.*/grid $g quad \1 ms/"; done
  (cd variants/mi1 && EPI4_STAGES=44 timeout 120 python tools/run_search.py 2>&1 | tail -1 | sed "s/best.*quad \([0-9.]*\) ms.*/mi1-44 quad \1 ms/")
  (cd variants/mi1 && timeout 120 python tools/run_search.py 2>&1 | tail -1 | sed "s/best.*quad \([0-9.]*\) ms.*/mi1-53 quad \1 ms/")
done
