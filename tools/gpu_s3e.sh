export KTILER_STAGE_POINTWISE=1
timeout 300 python tools/timeline.py --configs '[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":1.0,"exec_mode":"dag","discard":true,"window":2,"resident_budget":true},{"kind":"budget","l2_fraction":0.25,"exec_mode":"dag","discard":true,"window":4,"resident_budget":true}]' --out gpurun_out/tl_s3e.npz 2>&1 | tail -40
