python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 python -m pytest tests -q -m gpu -p no:cacheprovider 2>&1 | grep -E "^FAILED|^E  |passed|failed" | head -20
