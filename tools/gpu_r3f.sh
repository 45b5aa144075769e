#!/bin/bash
for c in 1 2 3 4 6 8; do BANDLU_TRFS_CHUNKS=$c timeout 120 python tools/time_chunks.py; done
for c in 1 2 4; do BANDLU_TRFS_CHUNKS=$c timeout 120 python tools/time_chunks.py 10000 50 10 10; done
for c in 1 2 4; do BANDLU_TRFS_CHUNKS=$c timeout 120 python tools/time_chunks.py 10000 256 1 1; done
