MAGIS_GEN_DEBUG=1 timeout 300 python scripts/gen_time.py c2 c5 2>&1 | tail -12
