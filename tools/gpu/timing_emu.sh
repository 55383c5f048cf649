# PSIM_TIMING timelines (CTA 0, step 900) at G=1 and at the G=8 per-GPU slice, plus per-GPU shares at G=2/4/8
bash tools/gpu/timing6.sh
bash tools/gpu/emu.sh
