#!/bin/bash
# e2e step-loop A/B of libdgr variants (scratch/e2e_probe.py per lib)
for lib in "$@"; do echo "$lib"; DGR_LIB=$lib python scratch/e2e_probe.py 2>&1 | tail -2; done
