cd /root/repo
SKIPS="0 1 2 3 8" timeout -s KILL 300 python tools/stage_probe.py caffenet_conv2:fwd caffenet_conv2:bwd_data caffenet_conv4:fwd caffenet_conv4:bwd_filter caffenet_conv3:bwd_data 2>&1 | tail -8
