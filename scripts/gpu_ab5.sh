for r in 1 2; do for v in 0 cf cf2 cs2 cf4 cfcta; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  line="$v $r"
  for w in tdes mm nop mb; do
    timeout 300 python bench.py --workload $w --quick --no-cpu --no-naive --steps 5 2>/dev/null | tail -1 > gpurun_out/ab5_${w}_${v}_$r.json
    line="$line $w=$(python -c "import json;d=json.load(open('gpurun_out/ab5_${w}_${v}_$r.json'));print(round(d['value']/1e6,2))")"
  done
  echo $line
done; done
export PAGODA_LIB=$PWD/build/variants/libpagoda_vcf4.so
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_runtime.py -q -x -k "not full_size" 2>&1 | tail -1
export PAGODA_LIB=$PWD/build/variants/libpagoda_vcfp.so
timeout 300 python scripts/probe_prof.py > gpurun_out/prof_cf.json 2>&1
