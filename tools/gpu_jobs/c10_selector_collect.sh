# re-collect selector training data with frag3 (training tensors only; never BASELINE shapes)
mkdir -p gpurun_out
timeout 2400 python tools/train_selector.py collect --count 260 --seed 11 --out gpurun_out/selector_train_frag3.jsonl > gpurun_out/c10_collect.log 2>&1
echo collect_exit=$?
wc -l gpurun_out/selector_train_frag3.jsonl
