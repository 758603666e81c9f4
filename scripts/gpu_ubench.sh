#!/bin/bash
mkdir -p gpurun_out
./scripts/ubench | tee gpurun_out/ubench.txt
