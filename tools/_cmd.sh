make -s all > /dev/null 2>&1
for G in 0 1 2; do timeout 300 python tools/relay_var.py google8_dgx1 $G; done
timeout 300 python tools/relay_var.py google8_ring 0
