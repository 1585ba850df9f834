# f2: stash tests and the VGG16 stash measurement (arena vs exact-size), b64
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_stash.py -x -q -p no:cacheprovider 2>&1 | tail -3
for mode in "" "--no-arena"; do
timeout 900 python scripts/mfr_vgg16.py --batch 64 --lossless $mode --json gpurun_out/f2_lossless$mode.json > gpurun_out/f2_lossless$mode.log 2>&1
python -c "import json,sys; d=json.load(open('gpurun_out/f2_lossless$mode.json')); print('$mode', d['baseline']['ms_per_step'], d['gist']['ms_per_step'], d['gist']['stash_bytes'], d['baseline']['stash_bytes'], d.get('mfr_peak'), d.get('ssdc_stash'))" || tail -5 gpurun_out/f2_lossless$mode.log
done
timeout 900 python scripts/mfr_vgg16.py --batch 64 --bits 16 --json gpurun_out/f2_dpr16.json > gpurun_out/f2_dpr16.log 2>&1; python -c "import json; d=json.load(open('gpurun_out/f2_dpr16.json')); print('dpr16', d['baseline']['ms_per_step'], d['gist']['ms_per_step'], d.get('mfr_peak'), d.get('ssdc_stash'))" || tail -5 gpurun_out/f2_dpr16.log
