# Round-2 gpurun helper: build, GPU tests, smoke, bench lines, measured shared-memory peak.
# TAG names the outputs; WORKLOADS / TESTS / SMOKE / SMEM / NCU select the parts.
set -u
TAG=${TAG:-r02}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/gpu_$TAG.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
if [ "${SMEM:-0}" = 1 ]; then
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/smem_peak tools/smem_peak.cu && \
    timeout 120 ./tools/smem_peak > gpurun_out/smem_peak_$TAG.txt 2>&1
fi
if [ "${TESTS:-1}" = 1 ]; then
  timeout ${TEST_TIMEOUT:-1800} python -m pytest tests -m gpu -q -x ${PYTEST_ARGS:-} > gpurun_out/pytest_gpu_$TAG.log 2>&1
  echo "pytest exit $?" >> gpurun_out/pytest_gpu_$TAG.log
fi
if [ "${SMOKE:-1}" = 1 ]; then
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
  echo "smoke exit $?" >> gpurun_out/smoke_$TAG.log
fi
for w in ${WORKLOADS:-C2a}; do
  timeout 900 python bench.py --workload $w ${BENCH_ARGS:-} > gpurun_out/bench_${TAG}_$w.log 2>&1
  tail -1 gpurun_out/bench_${TAG}_$w.log > gpurun_out/bench_${TAG}_$w.jsonl
done
if [ "${NCU:-0}" = 1 ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
      --log-file gpurun_out/launches_$TAG.csv \
      python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline ${NCU_BENCH_ARGS:-} > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KERNEL:-tile_reduce_kernel} -s 1 -c 1 \
      -o gpurun_out/prof_$TAG -f \
      python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline ${NCU_BENCH_ARGS:-} > gpurun_out/ncu_full_$TAG.log 2>&1
fi
echo done
