# usage: mp.sh model size transport port -> runs 2-process mp_check with a hard kill
timeout -s KILL 150 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=$4 tools/mp_check.py $1 $2 $3 > gpurun_out/mp_$1_$3.txt 2>&1
echo "mp rc=$?"; grep -v Warn gpurun_out/mp_$1_$3.txt | grep -E "rank|hios|Error|error" | head -20
