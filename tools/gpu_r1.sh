set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 600 python bench.py > gpurun_out/bench1.json 2> gpurun_out/bench1.err; echo bench_rc=$?
HIOS_NCU=1 timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu1.out 2>&1; echo ncu1_rc=$?
HIOS_NCU=1 timeout 900 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:conv_tc -s 6 -c 2 -o gpurun_out/prof_conv python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu2.out 2>&1; echo ncu2_rc=$?
tail -c 3000 gpurun_out/bench1.json; tail -20 gpurun_out/bench1.err
