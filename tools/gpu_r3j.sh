#!/bin/bash
for s in 2 3 4 6; do for c in 32 64 128 256; do
  BANDLU_HOST_STREAMS=$s BANDLU_HOST_CHUNK_MB=$c timeout 120 python tools/e2e_probe.py C3 3
done; done
