python -c "import __graft_entry__ as g; g.build()"
timeout 100 python tools/occ_debug.py 2>&1 | tail -14
