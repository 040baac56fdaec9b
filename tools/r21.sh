STF_GRAPH=0 timeout 300 python tools/timeline.py 8192 1024 dev 20 | grep "^k=\|device"
timeout 300 python tools/timeline.py 8192 1024 dev 20 | grep "^k=\|device"
