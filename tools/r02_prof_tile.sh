# one ncu --set full capture of tile_reduce_kernel (C2a by default) on the current build
set -u
TAG=${TAG:-r02p}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_reduce_kernel -s 3 -c 1 \
    -o gpurun_out/prof_tile_$TAG -f python bench.py --workload ${W:-C2a} --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/prof_$TAG.log 2>&1
echo done
