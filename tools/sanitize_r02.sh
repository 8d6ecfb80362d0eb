# round-2 (session 2) sanitizer runs on tools/race_tile.py: tile scan (summary and pattern paths,
# float 64-KiB and int32 tiles), 2x4x4-bricked cube, query-chunked fact-table scan
set -u
mkdir -p gpurun_out
python tools/race_tile.py > gpurun_out/san_plain_r02s2.txt 2>&1
for tool in memcheck synccheck racecheck; do
  timeout 1500 compute-sanitizer --tool $tool python tools/race_tile.py > gpurun_out/san_${tool}_r02s2.txt 2>&1
done
echo done
