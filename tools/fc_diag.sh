for L in fc6 fc7 fc8; do timeout 120 python tools/fc_diag.py $L 1 256 2>&1 | tail -2; done
