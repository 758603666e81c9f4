#!/bin/bash
mkdir -p gpurun_out
(./scripts/ubench; ./scripts/ubench_step) 2>&1 | tee gpurun_out/ubench.txt
