# packed 16-byte records for N >= 4: GPU suite + 4-way configs
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/c7_pytest.log 2>&1; echo pytest_exit=$?
tail -3 gpurun_out/c7_pytest.log
for c in deli4d flickr4d enron nips uber; do
  timeout 400 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/c7_f3pk_$c.json 2>gpurun_out/c7_f3pk_$c.err
done
echo done
