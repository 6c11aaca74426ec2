#!/bin/bash
# ncu launch list + one --set full capture (kernel regex $KREGEX) of one layer-pass (tools/pass_run.py)
cd "$(dirname "$0")"
mkdir -p gpurun_out
SPEC=${SPEC:-caffenet_conv1:bwd_filter}
TAGN=${TAG:-pass}
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launch_${TAGN}.csv python tools/pass_run.py $SPEC 3 ${WL:-4} > gpurun_out/ncu_${TAGN}_l.log 2>&1
echo "launch rc=$?"; python tools/launch_table.py gpurun_out/launch_${TAGN}.csv 2>&1 | tail -15
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-hwgrad} -s ${NSKIP:-1} -c 1 -o gpurun_out/prof_${TAGN} -f python tools/pass_run.py $SPEC 3 ${WL:-4} > gpurun_out/ncu_${TAGN}_f.log 2>&1
echo "full rc=$?"; tail -2 gpurun_out/ncu_${TAGN}_f.log
