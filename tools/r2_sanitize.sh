#!/bin/bash
# compute-sanitizer logs (racecheck, synccheck, memcheck, initcheck) for every kernel family,
# and the st27 step-by-three loop A/B against the parity tests
mkdir -p gpurun_out/san
export PYTHONUNBUFFERED=1
python -c "import oracle; oracle.build()"
for tool in memcheck racecheck synccheck initcheck; do
  for w in ${WHICH:-st7 st13 st27 lbm}; do
    timeout 1200 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
      python tools/sanitize_driver.py $w > gpurun_out/san/${tool}_${w}.log 2>&1
    echo "$tool $w rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|FAILURES' gpurun_out/san/${tool}_${w}.log | tr '\n' ' ')"
  done
done
ST35D_LIB=build/ab/step3/libst35d.so timeout 900 python -m pytest tests/test_gpu_st27.py -q -x > gpurun_out/san/st27_step3.log 2>&1
echo "st27 step-by-three loop: $(tail -1 gpurun_out/san/st27_step3.log)"
timeout 900 python -m pytest tests/test_gpu_st27.py -q -x > gpurun_out/san/st27_product.log 2>&1
echo "st27 product: $(tail -1 gpurun_out/san/st27_product.log)"
