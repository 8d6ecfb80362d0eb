# Round-2 evidence in one gpurun call: GPU tests, smoke, per-kernel DRAM bytes + instructions (traffic.sh),
# launch list, ncu --set full of the dominant kernels, bench lines of every workload with CPU baselines.
set -u
TAG=${TAG:-r02full}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/gpu_$TAG.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
if [ "${TESTS:-1}" = 1 ]; then
  timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu_$TAG.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke exit $?" >> gpurun_out/smoke_$TAG.log
fi
if [ "${TRAFFIC:-1}" = 1 ]; then
  # per-launch DRAM bytes + instructions first, so that the bench lines below use this build's counts
  WORKLOADS="${TRAFFIC_W:-C2a C2b C3 C4 C5 T C1}" timeout 1500 bash tools/traffic.sh
  python tools/traffic_json.py > gpurun_out/traffic_json_$TAG.log 2>&1
fi
for w in ${WORKLOADS:-C2a C2b C3 C4 C5 T R C1}; do
  timeout 900 python bench.py --workload $w ${BENCH_ARGS:-} > gpurun_out/bench_${TAG}_$w.log 2>&1
  tail -1 gpurun_out/bench_${TAG}_$w.log > gpurun_out/bench_${TAG}_$w.jsonl
done
if [ "${EXTRA:-1}" = 1 ]; then
  timeout 600 python bench.py --workload C1 --graph --no-cpu-baseline > gpurun_out/bench_${TAG}_C1g.log 2>&1; tail -1 gpurun_out/bench_${TAG}_C1g.log > gpurun_out/bench_${TAG}_C1g.jsonl
  timeout 600 python bench.py --workload C3 --no-cpu-baseline --stream-batch 4096 --e2e-steps 3 > gpurun_out/bench_${TAG}_C3s.log 2>&1; tail -1 gpurun_out/bench_${TAG}_C3s.log > gpurun_out/bench_${TAG}_C3s.jsonl
fi
if [ "${NCU:-1}" = 1 ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
      --log-file gpurun_out/launches_$TAG.csv \
      python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_reduce_kernel -s 3 -c 1 \
      -o gpurun_out/prof_tile_$TAG -f python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:table_scan_kernel -s 3 -c 1 \
      -o gpurun_out/prof_table_$TAG -f python bench.py --workload T --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:brick_reduce_kernel -s 3 -c 1 \
      -o gpurun_out/prof_brick_$TAG -f python bench.py --workload C5 --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
fi
echo done
