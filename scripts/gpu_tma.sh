#!/bin/bash
for m in 2 1 0; do for s in 1024 1040; do timeout 30 ./scripts/tma_probe $s 1 $m; done; done
