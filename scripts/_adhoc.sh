cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout -s KILL 900 python -m pytest tests/test_gpu_parity.py -q -x -k "halo_dgrad or mixed or exact_integer or samples_in_flight_invariance or rounding_emulated" -p no:cacheprovider 2>&1 | tail -15
export WL=4
for P in fwd bwd_filter bwd_data; do timeout -s KILL 300 python tools/pass_time.py caffenet_conv1:$P fp32 '{}' '{"fp32_split":0}' 2>&1 | tail -2; done
timeout -s KILL 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e --no-extra-modes 2>&1 | tail -1 | cut -c1-2600
