#!/bin/bash
# round evidence on one B200 (run under gpurun): GPU tests, smoke, the default
# bench line, the reference arm, the ncu launch list of one bench step (conv
# traffic), ncu --set full of the top kernels, Fig. 1/2 analog.  Every step has
# a hard timeout and writes to files (no pipes that could outlive a killed step).
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1 || { echo build failed; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout -s KILL 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu.txt
timeout -s KILL 300 python __graft_entry__.py smoke > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?"
T0=$(date +%s); timeout -s KILL 1200 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; echo "bench rc=$? wall=$(( $(date +%s) - T0 ))s"
T0=$(date +%s); timeout -s KILL 900 python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "ref rc=$? wall=$(( $(date +%s) - T0 ))s"
HIOS_NCU=1 timeout -s KILL 900 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --sweep "" > gpurun_out/ncu1.out 2>&1; echo "ncu list rc=$?"
python tools/ncu_summary.py gpurun_out/launches.csv > gpurun_out/launches_summary.txt 2>&1
python tools/conv_traffic.py gpurun_out/launches.csv inception_v3_1024 gpurun_out > gpurun_out/conv_traffic.txt 2>&1
HIOS_NCU=1 timeout -s KILL 900 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:conv_tc -s 4 -c 3 -o gpurun_out/full_conv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --sweep "" > gpurun_out/ncu2.out 2>&1; echo "ncu full rc=$?"
HIOS_NCU=1 timeout -s KILL 900 ncu --profile-from-start off --set full --clock-control none -k regex:pool -c 2 -o gpurun_out/full_pool python bench.py --steps 1 --warmup 3 --no-cpu-baseline --sweep "" > gpurun_out/ncu3.out 2>&1; echo "ncu pool rc=$?"
python tools/ncu_report.py gpurun_out/full_conv.ncu-rep gpurun_out/full_pool.ncu-rep > gpurun_out/ncu_full_summary.txt 2>&1

head -14 gpurun_out/launches_summary.txt
tail -c 1200 gpurun_out/bench_full.json
