# Session-4 follow-up: build, GPU tests, then A/B of the fused small-batch planner on C1
# (abvar/head.so = the previous cube.cu) with and without CUDA graphs.
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_s4b.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_r01s4b.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu_r01s4b.log
for rep in 1 2; do
  for v in head new; do
    if [ $v = head ]; then env="OLAP_LIB=abvar/head.so"; else env=""; fi
    for g in "" "--graph"; do
      env $env timeout 300 python bench.py --no-cpu-baseline --workload C1 --e2e-steps 1 $g 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C1 $v $g', round(d['value']), d['ms_per_step'], d.get('gpu_launches'))" >> gpurun_out/ab_c1.txt 2>&1
    done
  done
done
timeout 600 python bench.py --workload C1 > gpurun_out/bench_r01s4b_C1.log 2>&1; tail -1 gpurun_out/bench_r01s4b_C1.log > gpurun_out/bench_r01s4b_C1.jsonl
echo s4bdone
