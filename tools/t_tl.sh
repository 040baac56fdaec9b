#!/bin/bash
timeout 300 python tools/timeline.py 32768 1024 host 40
timeout 300 python tools/timeline.py 32768 1024 dev 40
timeout 300 python tools/timeline.py 8192 1024 dev 20
