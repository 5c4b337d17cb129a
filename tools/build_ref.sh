#!/bin/bash
# Build commit REV (default HEAD) in a scratch worktree and copy its library here as libeirene_NAME.so (A/B baseline)
REV=${1:-HEAD}; NAME=${2:-head}
W=/tmp/eirene_wt_$NAME
git worktree remove --force $W 2>/dev/null; rm -rf $W
git worktree add -f $W $REV -q && (cd $W && python -m paper_conf_ppopp_zhangz0lzl23_b200.build > /tmp/eirene_wt_$NAME.log 2>&1) \
  && cp $W/paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_$NAME.so
git worktree remove --force $W
ls -la paper_conf_ppopp_zhangz0lzl23_b200/libeirene_$NAME.so
