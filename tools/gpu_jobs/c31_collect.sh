# selector training data with the L2-tiled classes (7-9): small/medium and large random tensors
mkdir -p gpurun_out/c31
timeout 2000 python tools/train_selector.py collect --count 160 --seed 31 --prefix trainS --seed-base 31000000 --out gpurun_out/c31/train_small.jsonl > gpurun_out/c31/collect_small.log 2>&1; echo small_exit=$?
timeout 2600 python tools/train_selector.py collect --count 90 --seed 32 --prefix trainL --seed-base 32000000 --nnz-log10 7.5,8.2 --dims-log10 4.0,7.3 --out gpurun_out/c31/train_large.jsonl > gpurun_out/c31/collect_large.log 2>&1; echo large_exit=$?
wc -l gpurun_out/c31/*.jsonl
