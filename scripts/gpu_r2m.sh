cd "$(dirname "$0")/.."
for L in caffenet_conv3:bwd_data caffenet_conv5:fwd caffenet_conv5:bwd_data caffenet_conv3:fwd caffenet_conv4:fwd caffenet_conv4:bwd_data; do
  echo $L; WL=4 python tools/pass_time.py $L fp32 '{}' '{"tile_units":3}' '{"tile_units":4}' '{"tile_units":6}' '{"cta_pairs":0}' '{"cta_pairs":0,"tile_units":6}'
done
