#!/bin/bash
# validation of the committed default after the GZKP_CANON experiment: MSM / variant suites and the default bench line
OUT=${OUT:-gpurun_out/val}
mkdir -p $OUT
timeout 1500 python -m pytest tests/test_gpu_msm.py tests/test_gpu_variants.py tests/test_gpu_large.py tests/test_gpu_g2.py -m gpu -q -x -rfE -p no:cacheprovider > $OUT/pytest.txt 2>&1
tail -n2 $OUT/pytest.txt
timeout 400 python bench.py > $OUT/default.json 2> $OUT/default.err
python tools/summ.py $OUT/default.json
