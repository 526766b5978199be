# AlexNet fc6 / fc7 at B=256 in isolation: planner default vs A addressed as
# rectangle tiles (PCNN_AMODE=rect) and operand stage counts (PCNN_STAGES).
for L in fc6 fc7; do
  printf "default: "; timeout 60 python tools/one_layer.py $L 256 30 2>&1 | tail -1
  printf "rect: "; PCNN_AMODE=rect timeout 60 python tools/one_layer.py $L 256 30 2>&1 | tail -1
  for st in 2 3 4; do
    printf "stages=$st: "; PCNN_STAGES=$st timeout 60 python tools/one_layer.py $L 256 30 2>&1 | tail -1
  done
done
