mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q --timeout 300 -k "link_probe or wide_rank" > gpurun_out/t6_focus.log 2>&1; echo "rc=$?" >> gpurun_out/t6_focus.log
timeout 600 python scripts/profile_links.py --out gpurun_out/links_r02.json > gpurun_out/t6_links.log 2>&1
