# Per-CTA SSDC-encode timelines (needs var/libgist_trace.so built with -DGIST_SSDC_TRACE) on three VGG16 map sizes.
for shp in 64x512x14x14 64x256x28x28 64x64x224x224; do timeout 120 python scripts/ssdc_trace.py 0.8 $shp 2>&1 | tail -9; done
