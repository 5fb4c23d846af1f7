python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python scripts/probe_busy.py mm tdes nop mb > gpurun_out/busy.json 2>&1; cat gpurun_out/busy.json
for w in tdes mm; do timeout 300 python bench.py --workload $w --quick --no-cpu --no-naive 2>/dev/null | tail -1 > gpurun_out/q_$w.json; python -c "import json;d=json.load(open('gpurun_out/q_$w.json'));print('$w',d['value']/1e6)"; done
