python __graft_entry__.py > /dev/null 2>&1
for a in "--streams 1" "--streams 2" "--streams 4" "--streams 8" "--streams 4 --batch 262144"; do
  timeout 300 python bench.py --steps 400 --warmup 10 --no-e2e --no-cpu --search-budget 0 $a 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; print('$a', round(d['value']/1e9,3), 'Gcfg/s frac', round(r['frac'],3))"
done
