#!/bin/bash
# fixed-point sequence-conv wgrads, cv_c3 / nlp_c3 full-size goldens
set -x
timeout 1500 python -m pytest -q -x -s tests/test_gpu_parity.py -k "nlp" 2>&1 | grep -v "^$" | tail -12
timeout 1500 python -m pytest -q -x -s tests/test_gpu_spos.py -k "cv_c3" 2>&1 | grep -v "^$" | tail -8
