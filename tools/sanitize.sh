mkdir -p gpurun_out
K="brick_shapes or brick_every or brick_empty or brick_virtual or tile_and_item or small_boxes_take or c1_full or warp_items_large_batches and 64"
timeout 1500 compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_brick.py tests/test_gpu_tiles.py tests/test_gpu_parity.py -m gpu -q -k "brick_shapes or brick_every or brick_empty or brick_virtual or tile_and_item or c1_full" > gpurun_out/san_memcheck_s3.txt 2>&1
timeout 1500 compute-sanitizer --tool racecheck python -m pytest tests/test_gpu_brick.py tests/test_gpu_tiles.py -m gpu -q -k "brick_every or brick_empty or tile_and_item" > gpurun_out/san_racecheck_s3.txt 2>&1
timeout 1500 compute-sanitizer --tool synccheck python -m pytest tests/test_gpu_brick.py tests/test_gpu_tiles.py -m gpu -q -k "brick_every or brick_empty or tile_and_item" > gpurun_out/san_synccheck_s3.txt 2>&1
