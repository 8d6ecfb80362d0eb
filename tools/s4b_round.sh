# Session-4 follow-up: GPU tests (with the planner-boundary parity test) and C1 after the revert.
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_s4b.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_r01s4b.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu_r01s4b.log
for rep in 1 2; do
  timeout 600 python bench.py --workload C1 > gpurun_out/bench_r01s4b_C1_$rep.log 2>&1; tail -1 gpurun_out/bench_r01s4b_C1_$rep.log > gpurun_out/bench_r01s4b_C1_$rep.jsonl
done
timeout 600 python bench.py --workload C1 --graph --no-cpu-baseline > gpurun_out/bench_r01s4b_C1g.log 2>&1; tail -1 gpurun_out/bench_r01s4b_C1g.log > gpurun_out/bench_r01s4b_C1g.jsonl
echo s4bdone
