python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tc or fusion" > gpurun_out/pytest_tc.log 2>&1; tail -3 gpurun_out/pytest_tc.log
for w in ${WORKLOADS:-tdes mm_tc mm mb}; do
  timeout 600 python bench.py --workload $w --no-e2e --no-cpu --steps 5 --warmup 3 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
  python -c "
import json;d=json.loads(open('gpurun_out/bench_$w.json').read().strip().splitlines()[-1])
print('$w',round(d['value']/1e6,2),'M/s',round(d['ms_per_step'],3),'ms',d['roofline']['resource'],round(d['roofline']['frac'],3),'naive',round(d.get('naive',{}).get('tasks_per_s',0)/1e6,3),'fused',{k:round(v/1e6,2) for k,v in d.get('static_fusion',{}).items() if 'per_s' in k},'batch',round(d.get('batching',{}).get('tasks_per_s',0)/1e6,2))" || tail -5 gpurun_out/bench_$w.err
done
