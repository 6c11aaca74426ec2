cd "$(dirname "$0")/.."
for W in 1 2 3; do MATH=fp32 WORKLOAD=$W python tools/plan_dump.py; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:igemm -s 3 -c 1 -o gpurun_out/prof_lenet_wgrad -f python bench.py --steps 1 --warmup 1 --workload 1 --math fp32 --no-cpu-baseline --no-e2e --no-graph --serial --no-extra-modes > /dev/null 2>&1
echo ncu $?
