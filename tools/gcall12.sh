mkdir -p gpurun_out
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 2400 bash tools/ab.sh \
  ext \
  "ext:LA_CLASSES=64x12,128x6,256x4,512x2,1024x1" \
  "ext:LA_CLASSES=64x12,128x8,256x3,512x2,1024x1" \
  "ext:LA_CLASSES=64x16,128x6,256x3,512x2,1024x1" \
  "ext:LA_CLASSES=64x12,128x6,256x3,512x2,1024x1;LA_SMALL_MASK=7" \
  "ext:LA_CLASSES=64x12,96x8,256x3,512x2,1024x1" > gpurun_out/ab7_c4.txt 2>&1
