#!/bin/bash
mkdir -p gpurun_out
timeout 300 ./tools/mb_ingest > gpurun_out/mb_ingest.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_attention.py tests/test_quant_variants.py -m gpu -q -p no:cacheprovider -x > gpurun_out/pytest_attn.log 2>&1
tail -3 gpurun_out/pytest_attn.log
