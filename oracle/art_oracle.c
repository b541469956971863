/*
 * oracle/art_oracle.c — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, single-threaded, pointer-based Adaptive Radix Tree, written from the
 * paper (CuART, Koppehel et al., ICPP'21 — /root/reference/PAPER.md, cited as
 * P:<line>) and from the ART definition the paper defers to (Leis et al. 2013,
 * ref. [17]).  It is the correctness oracle for the CUDA path
 * in paper_conf_icpp_koppehelggp21_b200/ and shares no code, header, table or
 * constant with it.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load it.
 *
 * What it computes (the plain definition):
 *   lookup(q)      = value stored for q, else OART_MISS (UINT64_MAX)
 *   update(batch)  = apply (k_i, v_i) for i = 0..n-1 IN ORDER, only for keys
 *                    already present ("replace the value stored for
 *                    certain keys"; P:143 the highest op index wins).
 *
 * Keys are byte strings of length 1..32 (compile-time maximum), compared
 * lexicographically; integer keys are fed as big-endian bytes (reading C2).
 * The key set must be prefix-free (reading C3); insert reports an error otherwise.
 *
 * ART as in [17]: inner nodes Node4 / Node16 (sorted key bytes + children),
 * Node48 (256-entry child index + 48 children), Node256 (direct array), grown
 * when full at 4 / 16 / 48 (P:100 names the node types; P:108 numbers them
 * 1=N4, 2=N16, 3=N48, 4=N256).  Path compression: every inner node stores its
 * FULL compressed prefix (pessimistic, no optimistic skipping).  Lazy
 * expansion: a key is stored in a leaf hung at the shallowest node where it is
 * unique.  Insert-only: no shrinking (structural delete is out of scope).
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OART_MAX_KEY 32
#define OART_MISS UINT64_MAX

enum { K_LEAF = 0, K_N4 = 1, K_N16 = 2, K_N48 = 3, K_N256 = 4 };

typedef struct onode {
    int kind;
} onode;

typedef struct {
    int kind;                       /* K_LEAF */
    uint32_t len;
    uint8_t key[OART_MAX_KEY];
    uint64_t value;
    uint64_t pending;               /* batch scratch: 1 + index of the last op on this leaf */
} oleaf;

typedef struct {
    int kind;
    uint32_t prefix_len;            /* full compressed-path length */
    uint8_t prefix[OART_MAX_KEY];   /* full compressed path (pessimistic) */
    uint32_t count;                 /* number of children */
} oinner;

typedef struct { oinner h; uint8_t keys[4];  onode* child[4];   } onode4;
typedef struct { oinner h; uint8_t keys[16]; onode* child[16];  } onode16;
typedef struct { oinner h; uint8_t index[256]; /* 0 = empty, else slot+1 */ onode* child[48]; } onode48;
typedef struct { oinner h; onode* child[256]; } onode256;

typedef struct oart {
    onode* root;
    uint64_t n_keys;
} oart;

/* ------------------------------------------------------------------ helpers */
static oleaf* new_leaf(const uint8_t* key, uint32_t len, uint64_t value) {
    oleaf* l = (oleaf*)calloc(1, sizeof(oleaf));
    l->kind = K_LEAF;
    l->len = len;
    memcpy(l->key, key, len);
    l->value = value;
    return l;
}

static int key_equal(const oleaf* l, const uint8_t* key, uint32_t len) {
    return l->len == len && memcmp(l->key, key, len) == 0;
}

/* Find the child slot for byte b (Leis [17] Fig./Alg. "findChild"). */
static onode** find_child(onode* n, uint8_t b) {
    switch (n->kind) {
    case K_N4: {
        onode4* x = (onode4*)n;
        for (uint32_t i = 0; i < x->h.count; i++)
            if (x->keys[i] == b) return &x->child[i];
        return NULL;
    }
    case K_N16: {
        onode16* x = (onode16*)n;
        for (uint32_t i = 0; i < x->h.count; i++)      /* plain linear search, no SIMD */
            if (x->keys[i] == b) return &x->child[i];
        return NULL;
    }
    case K_N48: {
        onode48* x = (onode48*)n;
        if (x->index[b] == 0) return NULL;
        return &x->child[x->index[b] - 1];
    }
    case K_N256: {
        onode256* x = (onode256*)n;
        return x->child[b] ? &x->child[b] : NULL;
    }
    }
    return NULL;
}

/* Insert (b -> child) into a node that has room, keeping N4/N16 keys sorted. */
static void add_child_sorted(uint8_t* keys, onode** child, uint32_t count, uint8_t b, onode* c) {
    uint32_t pos = 0;
    while (pos < count && keys[pos] < b) pos++;
    memmove(keys + pos + 1, keys + pos, count - pos);
    memmove(child + pos + 1, child + pos, (count - pos) * sizeof(onode*));
    keys[pos] = b;
    child[pos] = c;
}

/* Add child; grow N4->N16->N48->N256 when full ([17] "grow"). *ref is the
 * parent's pointer to n, replaced on growth. */
static void add_child(onode** ref, uint8_t b, onode* c) {
    onode* n = *ref;
    switch (n->kind) {
    case K_N4: {
        onode4* x = (onode4*)n;
        if (x->h.count < 4) { add_child_sorted(x->keys, x->child, x->h.count, b, c); x->h.count++; return; }
        onode16* g = (onode16*)calloc(1, sizeof(onode16));
        g->h = x->h; g->h.kind = K_N16;
        memcpy(g->keys, x->keys, 4);
        memcpy(g->child, x->child, 4 * sizeof(onode*));
        free(x);
        *ref = (onode*)g;
        add_child(ref, b, c);
        return;
    }
    case K_N16: {
        onode16* x = (onode16*)n;
        if (x->h.count < 16) { add_child_sorted(x->keys, x->child, x->h.count, b, c); x->h.count++; return; }
        onode48* g = (onode48*)calloc(1, sizeof(onode48));
        g->h = x->h; g->h.kind = K_N48;
        for (uint32_t i = 0; i < 16; i++) { g->child[i] = x->child[i]; g->index[x->keys[i]] = (uint8_t)(i + 1); }
        free(x);
        *ref = (onode*)g;
        add_child(ref, b, c);
        return;
    }
    case K_N48: {
        onode48* x = (onode48*)n;
        if (x->h.count < 48) {
            uint32_t slot = x->h.count;        /* insert-only: slots 0..count-1 are used */
            x->child[slot] = c;
            x->index[b] = (uint8_t)(slot + 1);
            x->h.count++;
            return;
        }
        onode256* g = (onode256*)calloc(1, sizeof(onode256));
        g->h = x->h; g->h.kind = K_N256;
        for (int k = 0; k < 256; k++) if (x->index[k]) g->child[k] = x->child[x->index[k] - 1];
        free(x);
        *ref = (onode*)g;
        add_child(ref, b, c);
        return;
    }
    case K_N256: {
        onode256* x = (onode256*)n;
        x->child[b] = c;
        x->h.count++;
        return;
    }
    }
}

static onode4* new_node4(const uint8_t* prefix, uint32_t prefix_len) {
    onode4* x = (onode4*)calloc(1, sizeof(onode4));
    x->h.kind = K_N4;
    x->h.prefix_len = prefix_len;
    memcpy(x->h.prefix, prefix, prefix_len);
    return x;
}

/* ------------------------------------------------------------------ insert */
/* Returns 0 on success, 1 if the key set would stop being prefix-free. */
static int insert_rec(oart* t, onode** ref, const uint8_t* key, uint32_t len, uint64_t value, uint32_t depth) {
    onode* n = *ref;
    if (n == NULL) { *ref = (onode*)new_leaf(key, len, value); t->n_keys++; return 0; }

    if (n->kind == K_LEAF) {
        oleaf* l = (oleaf*)n;
        if (key_equal(l, key, len)) { l->value = value; return 0; }   /* duplicate: last wins (C6) */
        /* lazy expansion undone: new N4 holding both leaves under their first
         * differing byte; its prefix is the common part after `depth`. */
        uint32_t p = 0;
        while (depth + p < len && depth + p < l->len && key[depth + p] == l->key[depth + p]) p++;
        if (depth + p >= len || depth + p >= l->len) return 1;        /* one key is a prefix of the other */
        onode4* x = new_node4(key + depth, p);
        onode* nx = (onode*)x;
        add_child(&nx, l->key[depth + p], n);
        add_child(&nx, key[depth + p], (onode*)new_leaf(key, len, value));
        *ref = nx;
        t->n_keys++;
        return 0;
    }

    oinner* h = (oinner*)n;
    /* pessimistic prefix check: compare the full stored prefix */
    uint32_t p = 0;
    while (p < h->prefix_len && depth + p < len && h->prefix[p] == key[depth + p]) p++;
    if (p < h->prefix_len) {
        if (depth + p >= len) return 1;                                  /* key ends inside the prefix */
        /* split the compressed path at p: new N4 with prefix[0..p) */
        onode4* x = new_node4(h->prefix, p);
        onode* nx = (onode*)x;
        uint8_t old_byte = h->prefix[p];
        memmove(h->prefix, h->prefix + p + 1, h->prefix_len - (p + 1));
        h->prefix_len -= p + 1;
        add_child(&nx, old_byte, n);
        add_child(&nx, key[depth + p], (onode*)new_leaf(key, len, value));
        *ref = nx;
        t->n_keys++;
        return 0;
    }
    depth += h->prefix_len;
    if (depth >= len) return 1;                                          /* key is a prefix of stored keys */
    onode** c = find_child(n, key[depth]);
    if (c) return insert_rec(t, c, key, len, value, depth + 1);
    add_child(ref, key[depth], (onode*)new_leaf(key, len, value));
    t->n_keys++;
    return 0;
}

/* ------------------------------------------------------------------ public API */
oart* oart_new(void) { return (oart*)calloc(1, sizeof(oart)); }

static void free_rec(onode* n) {
    if (!n) return;
    switch (n->kind) {
    case K_N4:   { onode4* x = (onode4*)n;     for (uint32_t i = 0; i < x->h.count; i++) free_rec(x->child[i]); break; }
    case K_N16:  { onode16* x = (onode16*)n;   for (uint32_t i = 0; i < x->h.count; i++) free_rec(x->child[i]); break; }
    case K_N48:  { onode48* x = (onode48*)n;   for (uint32_t i = 0; i < x->h.count; i++) free_rec(x->child[i]); break; }
    case K_N256: { onode256* x = (onode256*)n; for (int i = 0; i < 256; i++) free_rec(x->child[i]); break; }
    default: break;
    }
    free(n);
}

void oart_free(oart* t) { if (t) { free_rec(t->root); free(t); } }

/* 0 ok, 1 not prefix-free, 2 bad length, 3 reserved value */
int oart_insert(oart* t, const uint8_t* key, uint32_t len, uint64_t value) {
    if (len == 0 || len > OART_MAX_KEY) return 2;
    if (value == OART_MISS) return 3;
    return insert_rec(t, &t->root, key, len, value, 0);
}

/* Bulk insert of n keys laid out with a fixed stride (slots of `stride` bytes). */
int oart_insert_batch(oart* t, const uint8_t* keys, const uint8_t* lens, uint32_t fixed_len,
                      size_t stride, const uint64_t* values, size_t n) {
    for (size_t i = 0; i < n; i++) {
        uint32_t len = lens ? lens[i] : fixed_len;
        int rc = oart_insert(t, keys + i * stride, len, values[i]);
        if (rc) return rc;
    }
    return 0;
}

uint64_t oart_size(const oart* t) { return t->n_keys; }

/* Leis [17] lookup with pessimistic path compression; leaf compares length+bytes. */
uint64_t oart_lookup(const oart* t, const uint8_t* key, uint32_t len) {
    onode* n = t->root;
    uint32_t depth = 0;
    while (n) {
        if (n->kind == K_LEAF) {
            oleaf* l = (oleaf*)n;
            return key_equal(l, key, len) ? l->value : OART_MISS;
        }
        oinner* h = (oinner*)n;
        if (depth + h->prefix_len >= len) return OART_MISS;              /* query too short */
        if (memcmp(h->prefix, key + depth, h->prefix_len) != 0) return OART_MISS;
        depth += h->prefix_len;
        onode** c = find_child(n, key[depth]);
        if (!c) return OART_MISS;
        n = *c;
        depth += 1;
    }
    return OART_MISS;
}

void oart_lookup_batch(const oart* t, const uint8_t* keys, const uint8_t* lens, uint32_t fixed_len,
                       size_t stride, size_t n, uint64_t* out) {
    for (size_t i = 0; i < n; i++)
        out[i] = oart_lookup(t, keys + i * stride, lens ? lens[i] : fixed_len);
}

/* The same read-only loop split into `threads` contiguous slices, one POSIX thread
 * each (the all-core CPU baseline of SURVEY §8(d); lookups never write the tree,
 * so the slices are independent and the result equals oart_lookup_batch's). */
typedef struct {
    const oart* t; const uint8_t* keys; const uint8_t* lens; uint32_t fixed_len; size_t stride;
    size_t lo, hi; uint64_t* out;
} lookup_slice;

static void* lookup_slice_run(void* arg) {
    const lookup_slice* a = (const lookup_slice*)arg;
    for (size_t i = a->lo; i < a->hi; i++)
        a->out[i] = oart_lookup(a->t, a->keys + i * a->stride, a->lens ? a->lens[i] : a->fixed_len);
    return NULL;
}

int oart_lookup_batch_mt(const oart* t, const uint8_t* keys, const uint8_t* lens, uint32_t fixed_len,
                         size_t stride, size_t n, uint64_t* out, int threads) {
    if (threads < 1) threads = 1;
    if (threads > 1024) threads = 1024;
    pthread_t tid[1024];
    int created[1024];
    lookup_slice sl[1024];
    for (int k = 0; k < threads; k++) {
        sl[k] = (lookup_slice){t, keys, lens, fixed_len, stride, n * (size_t)k / (size_t)threads,
                               n * (size_t)(k + 1) / (size_t)threads, out};
        created[k] = k < threads - 1 && pthread_create(&tid[k], NULL, lookup_slice_run, &sl[k]) == 0;
        if (!created[k]) lookup_slice_run(&sl[k]);   /* the caller's thread takes the last slice */
    }
    for (int k = 0; k < threads; k++)
        if (created[k]) pthread_join(tid[k], NULL);
    return threads;
}

static oleaf* find_leaf(const oart* t, const uint8_t* key, uint32_t len) {
    onode* n = t->root;
    uint32_t depth = 0;
    while (n) {
        if (n->kind == K_LEAF) {
            oleaf* l = (oleaf*)n;
            return key_equal(l, key, len) ? l : NULL;
        }
        oinner* h = (oinner*)n;
        if (depth + h->prefix_len >= len) return NULL;
        if (memcmp(h->prefix, key + depth, h->prefix_len) != 0) return NULL;
        depth += h->prefix_len;
        onode** c = find_child(n, key[depth]);
        if (!c) return NULL;
        n = *c;
        depth += 1;
    }
    return NULL;
}

/* Sequential batch update: ops applied in index order, so the op
 * with the highest index wins per key; absent keys are a no-op (reading C6).
 * Reading C5: CUART_MISS is reserved (it is the lookup's "absent" answer, so it
 * can never be stored); an op carrying it is DROPPED -- a no-op, as if its key
 * were absent -- and counted in *rejected; the other ops of the batch apply.
 * Returns the number of applied ops that hit a stored key. */
int64_t oart_update_batch(oart* t, const uint8_t* keys, const uint8_t* lens, uint32_t fixed_len,
                          size_t stride, const uint64_t* values, size_t n, uint64_t* rejected) {
    int64_t hits = 0;
    uint64_t rej = 0;
    for (size_t i = 0; i < n; i++) {
        if (values[i] == OART_MISS) { rej++; continue; }
        oleaf* l = find_leaf(t, keys + i * stride, lens ? lens[i] : fixed_len);
        if (l) { l->value = values[i]; hits++; }
    }
    if (rejected) *rejected = rej;
    return hits;
}

/* ------------------------------------------------------------------ dumps */
typedef struct { uint8_t* keys; uint8_t* lens; uint64_t* vals; size_t n, cap; } inorder_ctx;

static void inorder_rec(onode* n, inorder_ctx* c) {
    if (!n) return;
    switch (n->kind) {
    case K_LEAF: {
        oleaf* l = (oleaf*)n;
        if (c->n < c->cap) {
            memset(c->keys + c->n * OART_MAX_KEY, 0, OART_MAX_KEY);
            memcpy(c->keys + c->n * OART_MAX_KEY, l->key, l->len);
            c->lens[c->n] = (uint8_t)l->len;
            c->vals[c->n] = l->value;
        }
        c->n++;
        return;
    }
    case K_N4:   { onode4* x = (onode4*)n;   for (uint32_t i = 0; i < x->h.count; i++) inorder_rec(x->child[i], c); return; }
    case K_N16:  { onode16* x = (onode16*)n; for (uint32_t i = 0; i < x->h.count; i++) inorder_rec(x->child[i], c); return; }
    case K_N48:  { onode48* x = (onode48*)n; for (int k = 0; k < 256; k++) if (x->index[k]) inorder_rec(x->child[x->index[k] - 1], c); return; }
    case K_N256: { onode256* x = (onode256*)n; for (int k = 0; k < 256; k++) if (x->child[k]) inorder_rec(x->child[k], c); return; }
    }
}

/* In-order (lexicographic) (key, len, value) list; returns the number of leaves. */
size_t oart_dump_inorder(const oart* t, uint8_t* keys32, uint8_t* lens, uint64_t* vals, size_t cap) {
    inorder_ctx c = { keys32, lens, vals, 0, cap };
    inorder_rec(t->root, &c);
    return c.n;
}

/* Pre-order structure records as a stream of int64:
 *   inner: kind(1..4), prefix_len, prefix bytes..., count, child bytes in key order...
 *   leaf : 0, len, key bytes..., value
 * Children are visited in key-byte order. */
typedef struct { int64_t* buf; size_t n, cap; } rec_ctx;
static void put(rec_ctx* c, int64_t v) { if (c->n < c->cap) c->buf[c->n] = v; c->n++; }

static void children_in_order(onode* n, uint8_t* bytes, onode** kids, uint32_t* cnt) {
    uint32_t k = 0;
    switch (n->kind) {
    case K_N4:   { onode4* x = (onode4*)n;   for (uint32_t i = 0; i < x->h.count; i++) { bytes[k] = x->keys[i]; kids[k++] = x->child[i]; } break; }
    case K_N16:  { onode16* x = (onode16*)n; for (uint32_t i = 0; i < x->h.count; i++) { bytes[k] = x->keys[i]; kids[k++] = x->child[i]; } break; }
    case K_N48:  { onode48* x = (onode48*)n; for (int b = 0; b < 256; b++) if (x->index[b]) { bytes[k] = (uint8_t)b; kids[k++] = x->child[x->index[b] - 1]; } break; }
    case K_N256: { onode256* x = (onode256*)n; for (int b = 0; b < 256; b++) if (x->child[b]) { bytes[k] = (uint8_t)b; kids[k++] = x->child[b]; } break; }
    }
    *cnt = k;
}

static void struct_rec(onode* n, rec_ctx* c) {
    if (!n) return;
    if (n->kind == K_LEAF) {
        oleaf* l = (oleaf*)n;
        put(c, 0); put(c, l->len);
        for (uint32_t i = 0; i < l->len; i++) put(c, l->key[i]);
        put(c, (int64_t)l->value);
        return;
    }
    oinner* h = (oinner*)n;
    uint8_t bytes[256]; onode* kids[256]; uint32_t cnt;
    children_in_order(n, bytes, kids, &cnt);
    put(c, h->kind); put(c, h->prefix_len);
    for (uint32_t i = 0; i < h->prefix_len; i++) put(c, h->prefix[i]);
    put(c, cnt);
    for (uint32_t i = 0; i < cnt; i++) put(c, bytes[i]);
    for (uint32_t i = 0; i < cnt; i++) struct_rec(kids[i], c);
}

/* Returns the number of int64 words needed; writes up to cap. */
size_t oart_dump_structure(const oart* t, int64_t* buf, size_t cap) {
    rec_ctx c = { buf, 0, cap };
    struct_rec(t->root, &c);
    return c.n;
}

/* Node counts by kind: out[0]=leaves, out[1..4]=N4,N16,N48,N256; out[5]=max depth (nodes). */
static void stats_rec(onode* n, uint64_t* out, uint64_t level) {
    if (!n) return;
    if (level > out[5]) out[5] = level;
    out[n->kind]++;
    if (n->kind == K_LEAF) return;
    uint8_t bytes[256]; onode* kids[256]; uint32_t cnt;
    children_in_order(n, bytes, kids, &cnt);
    for (uint32_t i = 0; i < cnt; i++) stats_rec(kids[i], out, level + 1);
}

void oart_stats(const oart* t, uint64_t out[6]) {
    memset(out, 0, 6 * sizeof(uint64_t));
    stats_rec(t->root, out, 1);
}

/* ------------------------------------------------------------------ deletes
 * Non-structural delete (§3.3): the key's leaf is removed and its
 * reference is dropped from the parent; nodes are NOT collapsed or shrunk. */
static void remove_child(onode* n, uint8_t b) {
    switch (n->kind) {
    case K_N4:
    case K_N16: {
        uint8_t* keys = n->kind == K_N4 ? ((onode4*)n)->keys : ((onode16*)n)->keys;
        onode** child = n->kind == K_N4 ? ((onode4*)n)->child : ((onode16*)n)->child;
        oinner* h = (oinner*)n;
        uint32_t pos = 0;
        while (pos < h->count && keys[pos] != b) pos++;
        if (pos == h->count) return;
        memmove(keys + pos, keys + pos + 1, h->count - pos - 1);
        memmove(child + pos, child + pos + 1, (h->count - pos - 1) * sizeof(onode*));
        h->count--;
        return;
    }
    case K_N48: {
        onode48* x = (onode48*)n;
        if (!x->index[b]) return;
        uint32_t slot = x->index[b] - 1, last = x->h.count - 1;
        x->index[b] = 0;
        if (slot != last) {                         /* keep slots 0..count-1 dense */
            for (int k = 0; k < 256; k++)
                if (x->index[k] == last + 1) { x->index[k] = (uint8_t)(slot + 1); break; }
            x->child[slot] = x->child[last];
        }
        x->child[last] = NULL;
        x->h.count--;
        return;
    }
    case K_N256: {
        onode256* x = (onode256*)n;
        if (x->child[b]) { x->child[b] = NULL; x->h.count--; }
        return;
    }
    }
}

/* Unlink the leaf of key (pessimistic walk); returns the unlinked leaf or NULL.
 * The leaf is not freed here (the caller may still hold pointers to it). */
static oleaf* unlink_leaf(oart* t, const uint8_t* key, uint32_t len) {
    onode* parent = NULL;
    uint8_t pbyte = 0;
    onode* n = t->root;
    uint32_t depth = 0;
    while (n) {
        if (n->kind == K_LEAF) {
            oleaf* l = (oleaf*)n;
            if (!key_equal(l, key, len)) return NULL;
            if (parent) remove_child(parent, pbyte);
            else t->root = NULL;
            t->n_keys--;
            return l;
        }
        oinner* h = (oinner*)n;
        if (depth + h->prefix_len >= len) return NULL;
        if (memcmp(h->prefix, key + depth, h->prefix_len) != 0) return NULL;
        depth += h->prefix_len;
        onode** c = find_child(n, key[depth]);
        if (!c) return NULL;
        parent = n;
        pbyte = key[depth];
        n = *c;
        depth += 1;
    }
    return NULL;
}

int oart_erase(oart* t, const uint8_t* key, uint32_t len) {
    oleaf* l = unlink_leaf(t, key, len);
    if (!l) return 0;
    free(l);
    return 1;
}

/* A batch of updates and deletes (updates replace values; a delete is
 * the same operation with a "nil" value).  Reading C17: every op
 * locates its key in the state BEFORE the batch (stage 1 of Fig. 6 is a lookup
 * over the unmodified tree); for each located key the op with the highest index
 * decides -- its value is stored, or, for a delete, the key is removed.  Ops on
 * keys absent before the batch are no-ops.  Reading C5: a non-delete op carrying
 * the reserved value CUART_MISS is dropped (it locates nothing, so it never wins)
 * and counted in *rejected.  Returns the number of ops that located their key. */
int64_t oart_apply_batch(oart* t, const uint8_t* keys, const uint8_t* lens, uint32_t fixed_len, size_t stride,
                         const uint64_t* values, const uint8_t* is_delete, size_t n, uint64_t* rejected) {
    uint64_t rej = 0;
    oleaf** at = (oleaf**)calloc(n ? n : 1, sizeof(oleaf*));
    int64_t hits = 0;
    for (size_t i = 0; i < n; i++) {                /* stage 1: locate on the pre-batch tree */
        if ((!is_delete || !is_delete[i]) && values && values[i] == OART_MISS) {
            at[i] = NULL;                           /* reading C5: dropped */
            rej++;
            continue;
        }
        at[i] = find_leaf(t, keys + i * stride, lens ? lens[i] : fixed_len);
        if (at[i]) hits++;
    }
    if (rejected) *rejected = rej;
    /* highest op index per leaf: later ops overwrite the leaf's pending mark */
    for (size_t i = 0; i < n; i++)
        if (at[i]) at[i]->pending = (uint64_t)i + 1;
    uint8_t* win = (uint8_t*)calloc(n ? n : 1, 1);
    for (size_t i = 0; i < n; i++)
        if (at[i] && at[i]->pending == (uint64_t)i + 1) win[i] = 1;
    for (size_t i = 0; i < n; i++)
        if (at[i]) at[i]->pending = 0;
    oleaf** dead = (oleaf**)calloc(n ? n : 1, sizeof(oleaf*));
    size_t nd = 0;
    for (size_t i = 0; i < n; i++) {                /* stage 2: winners apply */
        if (!win[i]) continue;
        if (is_delete && is_delete[i]) {
            oleaf* l = unlink_leaf(t, keys + i * stride, lens ? lens[i] : fixed_len);
            if (l) dead[nd++] = l;
        } else {
            at[i]->value = values[i];
        }
    }
    for (size_t i = 0; i < nd; i++) free(dead[i]);
    free(dead);
    free(win);
    free(at);
    return hits;
}
