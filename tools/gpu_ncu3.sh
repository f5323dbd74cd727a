#!/bin/bash
LAUNCHES=0 bash tools/gpu_ncu.sh
