# L2-tile revisit threshold: 0.25 (default) vs 0.5 / 0.75 on random sets 1, 2 and BASELINE hyper-sparse shapes
mkdir -p gpurun_out/c36
for r in 0.5 0.75; do
  SF_L2_MAX_REVISIT=$r BLOCK_MB=64 timeout 1500 python tools/l2tile_study.py random:16:1 > gpurun_out/c36/rand1_$r.jsonl 2>/dev/null
  SF_L2_MAX_REVISIT=$r BLOCK_MB=64 timeout 1500 python tools/l2tile_study.py random:12:2 > gpurun_out/c36/rand2_$r.jsonl 2>/dev/null
  SF_L2_MAX_REVISIT=$r BLOCK_MB=64 timeout 1500 python tools/l2tile_study.py nell1,deli4d,deli3d,flickr3d,flickr4d > gpurun_out/c36/base_$r.jsonl 2>/dev/null
done
BLOCK_MB=64 timeout 1500 python tools/l2tile_study.py random:12:2 > gpurun_out/c36/rand2_0.25.jsonl 2>/dev/null
wc -l gpurun_out/c36/*.jsonl
