cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/conv_micro.py 6e_1x7 7c_1x1 7c_3x3 5b_1x1 6e_1x1 5b_5x5 4a > gpurun_out/micro.txt 2>&1; echo "micro rc=$?"
cat gpurun_out/micro.txt | grep -v Warn
timeout 300 python tools/conv_trace.py 6e_1x7 7c_1x1 7c_3x3 5b_1x1 > gpurun_out/trace.txt 2>&1; echo "trace rc=$?"
grep -v Warn gpurun_out/trace.txt | head -120
timeout 900 python -m pytest tests -q -m gpu -k "fullsize" > gpurun_out/pytest_full.txt 2>&1; echo "pytest full rc=$?"
tail -3 gpurun_out/pytest_full.txt
timeout 900 python bench.py --sweep "" --steps 20 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -c 3000 gpurun_out/bench.json; tail -5 gpurun_out/bench.err
