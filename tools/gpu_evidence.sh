#!/bin/bash
# round evidence: GPU tests, smoke, conv traffic (ncu launch list), default
# bench line, reference arm, ncu --set full of the top kernels, per-op tables
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?"
HIOS_NCU=1 timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --sweep "" > gpurun_out/ncu1.out 2>&1; echo "ncu list rc=$?"
python tools/ncu_summary.py gpurun_out/launches.csv > gpurun_out/launches_summary.txt 2>&1
python tools/conv_traffic.py gpurun_out/launches.csv inception_v3_1024
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "ref rc=$?"
HIOS_NCU=1 timeout 900 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:conv_tc -s 4 -c 3 -o gpurun_out/full_conv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --sweep "" > gpurun_out/ncu2.out 2>&1; echo "ncu full rc=$?"
HIOS_NCU=1 timeout 900 ncu --profile-from-start off --set full --clock-control none -k regex:pool -c 2 -o gpurun_out/full_pool python bench.py --steps 1 --warmup 3 --no-cpu-baseline --sweep "" > gpurun_out/ncu3.out 2>&1; echo "ncu pool rc=$?"
python tools/ncu_report.py gpurun_out/full_conv.ncu-rep gpurun_out/full_pool.ncu-rep > gpurun_out/ncu_full_summary.txt 2>&1
bash tools/gpu_dump.sh inception_v3@1024 inception_v3@4096 > gpurun_out/op_tables.txt 2>&1
head -14 gpurun_out/launches_summary.txt; cat gpurun_out/ncu_full_summary.txt | cut -c1-300
tail -c 1500 gpurun_out/bench_full.json; tail -c 600 gpurun_out/bench_ref.json
