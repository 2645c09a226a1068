#!/bin/bash
cd /root/repo && python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -5
