#!/bin/bash
# biased sampler: parity of the register-path variants, then A/B (one position per lane, 32-bit rounds)
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
echo "== tests"; timeout 900 python -m pytest tests -m gpu -q -k "biased" 2>&1 | tail -3
echo "== ab"; VARIANTS="${VARIANTS:-main old nolane1 nor32}" ROUNDS=2 STEPS=100 EXTRA="--scheme biased" bash tools/ab_variants.sh
