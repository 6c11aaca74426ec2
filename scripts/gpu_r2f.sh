cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for W in 1 5; do
timeout -s KILL 600 ncu --metrics gpu__time_duration.sum,sm__cycles_elapsed.max,smsp__cycles_active.avg --clock-control none --csv \
  --log-file gpurun_out/launch_small_$W.csv python bench.py --steps 1 --warmup 1 --workload $W --math fp32 --no-cpu-baseline --no-e2e --no-graph --serial --no-extra-modes > /dev/null 2>&1
echo "wl $W rc=$?"
done
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:igemm -s 4 -c 1 -o gpurun_out/prof_lenet_fwd -f python bench.py --steps 1 --warmup 1 --workload 1 --math fp32 --no-cpu-baseline --no-e2e --no-graph --serial --no-extra-modes > /dev/null 2>&1
echo "full rc=$?"
