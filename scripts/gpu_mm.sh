O=gpurun_out/mm4; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "mm or fusion or naive or mix" > $O/t.log 2>&1; tail -1 $O/t.log
timeout 900 python -m pytest tests/test_gpu_workloads.py -m gpu -q -k "c5_small or mpe_small" > $O/t2.log 2>&1; tail -1 $O/t2.log
for w in mm mm_tc mix c5 mpe; do for i in 1 2; do timeout 300 python bench.py --workload $w --quick 2>/dev/null | tail -1 > $O/${w}_$i.json
python -c "import json;d=json.loads(open('$O/${w}_$i.json').read().strip().splitlines()[-1]);print('$w', round(d['value']/1e6,2))"; done; done
timeout 600 python bench.py --workload mm --no-cpu > $O/mm_full.json 2>/dev/null
python -c "import json;d=json.loads(open('$O/mm_full.json').read().strip().splitlines()[-1]);print('mm full', round(d['value']/1e6,2), d['static_fusion'])"
