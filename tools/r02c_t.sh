#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_packed_gpu.py tests/test_peer_exchange_gpu.py -q -p no:cacheprovider --timeout 300 -rf 2>&1 | tail -4
timeout 600 python bench.py --config C2 --force-dist --exchange peer --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>&1 | tail -1 | cut -c1-300
