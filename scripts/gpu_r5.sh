# GPU tests (incl. multi-producer and lifecycle), lifecycle probe, quick bench check.
mkdir -p gpurun_out/r5; O=gpurun_out/r5
timeout 1500 python -m pytest tests -m gpu -q -x > $O/pytest_gpu.log 2>&1
timeout 600 python scripts/probe_life.py nop mm tdes mix mb > $O/life.jsonl 2> $O/life.err
for w in tdes mm nop; do timeout 300 python bench.py --workload $w --quick > $O/b_$w.json 2>/dev/null; done
tail -3 $O/pytest_gpu.log; cat $O/life.jsonl; tail -3 $O/life.err
for w in tdes mm nop; do python -c "import json;d=json.loads(open('$O/b_$w.json').read().strip().splitlines()[-1]);print('$w',round(d['value']/1e6,2))"; done
