# L2-tile block sizes after the tile-walk change: BASELINE/Table III shapes + random set 1
mkdir -p gpurun_out/c35
BLOCK_MB=16,32,64,128 timeout 1500 python tools/l2tile_study.py nell1,deli4d,deli3d,flickr3d,flickr4d > gpurun_out/c35/base.jsonl 2> gpurun_out/c35/err1.txt
BLOCK_MB=16,32,64,128 timeout 1500 python tools/l2tile_study.py random:16:1 > gpurun_out/c35/rand1.jsonl 2> gpurun_out/c35/err2.txt
wc -l gpurun_out/c35/*.jsonl
