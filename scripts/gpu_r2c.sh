cd /root/repo
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "tracker or eq7_launch or stream_pool" 2>&1 | tail -5
for w in 1 3 4; do timeout 300 python bench.py --scheme pool --workload $w --steps 3 --warmup 1 2>&1 | tail -1 | cut -c1-900; done
PYTEST_ARGS="" timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -k "cfg8" 2>&1 | tail -3
timeout 300 python bench.py --workload 8 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/workloads/wl_8.json 2>gpurun_out/workloads/wl_8.err; echo wl8 rc=$?
SKIPS=12 TAG=fp32dg bash scripts/gpu_profile_fp32.sh > /dev/null 2>&1; echo prof rc=$?
