export PYTHONUNBUFFERED=1
for st in 10 30 300; do timeout 300 python bench.py --steps $st --warmup 3 --no-cpu-baseline --no-breakdown 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('steps $st: GEPS %.3f ms/step %.4f frac %.3f host %.4f' % (d['value']/1e9, d['ms_per_step'], d['roofline']['frac'], d['host_issue_ms_per_step']))"; done
for inst in 2 4 3; do ARGS="--instances $inst" VARIANTS=base REPS=2 bash tools/ab_bench.sh | sed "s/^/inst $inst /"; done
