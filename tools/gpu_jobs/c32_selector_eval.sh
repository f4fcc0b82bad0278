# retrained selector (10 classes incl. L2 tiles): held-out random sets, BASELINE-shape study, eval
mkdir -p gpurun_out/c32
timeout 1500 python tools/l2tile_study.py random:16:1 > gpurun_out/c32/rand1.jsonl 2> gpurun_out/c32/err1.txt
timeout 1500 python tools/l2tile_study.py random:12:2 > gpurun_out/c32/rand2.jsonl 2> gpurun_out/c32/err2.txt
timeout 1500 python tools/l2tile_study.py nell2,vast,enron,deli3d,flickr3d,flickr4d,nell1,deli4d > gpurun_out/c32/base.jsonl 2> gpurun_out/c32/err3.txt
timeout 1500 python tools/train_selector.py eval --configs nell2,deli4d,nell1,flickr3d,deli3d --out gpurun_out/c32/eval.jsonl > /dev/null 2> gpurun_out/c32/err4.txt
tail -2 gpurun_out/c32/err*.txt
wc -l gpurun_out/c32/*.jsonl
