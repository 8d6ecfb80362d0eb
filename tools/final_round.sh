# End-of-session evidence in one gpurun call: GPU tests, smoke, bench lines for every workload,
# per-kernel DRAM traffic (tools/traffic.sh), launch list and ncu --set full of the C2a and C5 kernels.
set -u
TAG=${TAG:-r01s3b}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
bash tools/traffic.sh
for w in C2a C2b C3 C4 C5 T R C1; do
  timeout 600 python bench.py --workload $w > gpurun_out/bench_${TAG}_$w.log 2>&1
  tail -1 gpurun_out/bench_${TAG}_$w.log > gpurun_out/bench_${TAG}_$w.jsonl
done
timeout 600 python bench.py --workload C5 --layout row --no-cpu-baseline > gpurun_out/bench_${TAG}_C5row.log 2>&1; tail -1 gpurun_out/bench_${TAG}_C5row.log > gpurun_out/bench_${TAG}_C5row.jsonl
timeout 600 python bench.py --workload C1 --graph --no-cpu-baseline > gpurun_out/bench_${TAG}_C1g.log 2>&1; tail -1 gpurun_out/bench_${TAG}_C1g.log > gpurun_out/bench_${TAG}_C1g.jsonl
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_reduce_kernel -s 1 -c 1 -o gpurun_out/prof_tile_$TAG -f \
    python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
echo done
