# Session-4 close: full GPU suite, smoke, T and C2a bench lines on the final code.
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_s4f.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_r01s4f.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu_r01s4f.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_r01s4f.log 2>&1
for w in T C2a; do
  timeout 600 python bench.py --workload $w > gpurun_out/bench_r01s4f_$w.log 2>&1; tail -1 gpurun_out/bench_r01s4f_$w.log > gpurun_out/bench_r01s4f_$w.jsonl
done
echo s4fdone
