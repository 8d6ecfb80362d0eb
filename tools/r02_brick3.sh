# brick3 (2 x 4 x 4) check: bricked parity tests, C5 full-size sample, C5 bench lines for both brick
# shapes, DRAM bytes per launch of brick_reduce_kernel for both
set -u
TAG=${TAG:-r02b3}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
timeout 900 python -m pytest tests/test_gpu_brick.py tests/test_gpu_mgpu.py -m gpu -q -x > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_$TAG.log
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "c5 or C5 or brick" > gpurun_out/pytest_c5_$TAG.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_c5_$TAG.log
for lay in brick brick3; do
  timeout 600 python bench.py --workload C5 --layout $lay --no-cpu-baseline > gpurun_out/bench_${TAG}_C5_$lay.log 2>&1
  tail -1 gpurun_out/bench_${TAG}_C5_$lay.log > gpurun_out/bench_${TAG}_C5_$lay.jsonl
  timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none \
      -k regex:brick_reduce --csv --log-file gpurun_out/traffic_${TAG}_$lay.csv \
      python bench.py --workload C5 --layout $lay --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
done
echo done
