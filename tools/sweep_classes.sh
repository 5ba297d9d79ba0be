for cfg in "64x12,128x6,256x3,256x2,512x1" "96x8,128x6,256x3,256x2,512x1" "128x6,192x4,256x3,256x2,512x1" "128x6,256x3,256x2,512x1,512x1"; do
  echo "CFG $cfg"
  LA_CLASSES=$cfg timeout 600 python tools/phase_profile.py > gpurun_out/ph.json 2>/dev/null
  python -c "
import json
d=json.load(open('gpurun_out/ph.json'))
t=0
for k,v in d.items(): t+=v['ms']; print('  ', k, v['ms'], v['ends'], v['builder_cycles_per_attempt'], v['inserts_per_attempt'])
print('  total', round(t,2))
"
done
