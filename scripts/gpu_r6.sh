# Full GPU suite on the tree (4 forwarders), A/B vs 1 forwarder, MM drain without the host (prespawn).
O=gpurun_out/r6; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x > $O/pytest_gpu.log 2>&1
tail -3 $O/pytest_gpu.log
VARS="0 fwd1" AB=r6 bash scripts/gpu_ab.sh
for w in mm nop tdes; do for i in 1 2; do
  timeout 300 python bench.py --workload $w --quick --prespawn 2>/dev/null | tail -1 > $O/pre_${w}_$i.json
  python -c "import json;d=json.loads(open('$O/pre_${w}_$i.json').read().strip().splitlines()[-1]);print('prespawn $w',round(d['value']/1e6,2))"
done; done
