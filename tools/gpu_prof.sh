# conv kernel deep-dive: halo parity, per-op real timings, ncu full on 4 conv launches
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "conv_parity" > gpurun_out/tp.log 2>&1; echo tp_rc=$?; tail -3 gpurun_out/tp.log
HIOS_DUMP=gpurun_out/op_times.json timeout 600 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bp.json 2> gpurun_out/bp.err; echo bp_rc=$?
for s in 4 6 40 80; do
HIOS_NCU=1 timeout 600 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:conv_tc -s $s -c 1 -o gpurun_out/pc_$s python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu_$s=$?
done
