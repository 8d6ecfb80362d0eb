mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_brick.py -q -x -m gpu > gpurun_out/brick_tests.log 2>&1; echo "exit $?" >> gpurun_out/brick_tests.log
for L in row brick; do
  timeout 300 python bench.py --workload C5 --layout $L --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 > gpurun_out/c5_$L.jsonl
done
timeout 300 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --clock-control none -k regex:"reduce_kernel" -c 4 python bench.py --workload C5 --layout brick --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > gpurun_out/c5_brick_ncu.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "c5_slice_bricked" > gpurun_out/brick_c5_test.log 2>&1; echo "exit $?" >> gpurun_out/brick_c5_test.log
