# one --set full capture of the MasterKernel on the 3DES workload (self-draining session)
# usage: bash scripts/ncu_tdes.sh <out-name> [workload]
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master -s 3 -c 1 -o gpurun_out/$1 \
  python bench.py --workload ${2:-tdes} --prespawn --steps 1 --warmup 3 --no-naive --no-cpu --quick > gpurun_out/$1.log 2>&1
