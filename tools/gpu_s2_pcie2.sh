#!/bin/bash
O=gpurun_out/s2c
mkdir -p $O
timeout 600 python tools/pcie_pattern.py $O/pcie_rows.json rows 2>&1 | tail -20
