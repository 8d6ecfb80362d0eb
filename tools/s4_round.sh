# Session-4 evidence: the final_round.sh set plus an ncu --set full capture of table_scan_kernel on T.
set -u
TAG=${TAG:-r01s4}
bash tools/final_round.sh
timeout 900 ncu --set full --clock-control none --import-source on -k regex:table_scan_kernel -s 1 -c 1 -o gpurun_out/prof_table_$TAG -f \
    python bench.py --workload T --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
echo s4done
