for g in 1 0; do for c in 1 2 4 8 16; do echo "GRAPH=$g CHUNKS=$c"; NITRO_RUN_HOST_GRAPH=$g NITRO_RUN_HOST_CHUNKS=$c timeout 300 python tools/e2e_probe.py 2>&1 | tail -4; done; done
