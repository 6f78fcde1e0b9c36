# quick perf loop: conv parity, bench (no CPU leg), ncu launch list of the timed region
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "conv_parity or tiny or zoo" > gpurun_out/tq.log 2>&1; echo tq_rc=$?; tail -3 gpurun_out/tq.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bq.json 2> gpurun_out/bq.err; echo bq_rc=$?
HIOS_NCU=1 timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/lq.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --sweep "" > /dev/null 2>&1; echo ncu_rc=$?
python tools/ncu_summary.py gpurun_out/lq.csv
python -c "import json; d=json.load(open('gpurun_out/bq.json')); print('ms', d['value'], 'conv', d['roofline']['achieved'], 'cp', d['critical_path'], 'refs', d['single_gpu_refs'], 'e2e', d['e2e']['value'])"
tail -5 gpurun_out/bq.err
