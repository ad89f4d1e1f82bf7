/*
 * datagen/ssbgen.c -- seeded, counter-based synthetic SSB / TPC-H column generator.
 *
 * This module is SHARED INPUT INFRASTRUCTURE: both the oracle (oracle/) and the
 * product (paper_conf_sigmod_bressft16_b200/) consume its columns.  It holds none
 * of the method's arithmetic (no selection, join, gather or aggregation); it only
 * produces base-table columns and their string dictionaries.
 *
 * Why synthetic: the paper evaluates on SSB [28] and
 * TPC-H but ships no data, and there is no network for dbgen.
 * The recipe is SURVEY.md 8(c).2 (readings O2, O3, O4, O6, O12, O21 in DESIGN.md).
 *
 * Counter-based: every value is a pure function H(seed, table, draw, index), so any
 * row range can be regenerated bit-identically by any thread, process or shard.
 *
 * Widths (reading O3): keys, dates and dictionary codes are int32; measures int64.
 * Dictionaries are order-preserving (reading O4): code = rank of the string in the
 * bytewise-sorted list of distinct strings.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <stdio.h>
#include <math.h>

/* ------------------------------------------------------------------ hashing */
static inline uint64_t mix64(uint64_t x) { /* splitmix64 finaliser */
  x ^= x >> 30; x *= 0xBF58476D1CE4E5B9ULL;
  x ^= x >> 27; x *= 0x94D049BB133111EBULL;
  x ^= x >> 31; return x;
}
/* H(seed, table, draw, i): the single source of randomness. */
static inline uint64_t H(uint64_t seed, uint32_t table, uint32_t draw, uint64_t i) {
  uint64_t s = mix64(seed + 0x9E3779B97F4A7C15ULL * (uint64_t)(1 + table * 256u + draw));
  return mix64(s ^ (i * 0xD1B54A32D192ED03ULL + 0x632BE59BD9B4E019ULL));
}
uint64_t ddqgen_hash(uint64_t seed, uint32_t table, uint32_t draw, uint64_t i) {
  return H(seed, table, draw, i);
}

/* ------------------------------------------------------------- dictionaries */
enum {
  DICT_NATION = 0, DICT_REGION, DICT_CITY, DICT_MFGR, DICT_CATEGORY, DICT_BRAND1,
  DICT_YEARMONTH, DICT_MKTSEGMENT, DICT_ORDERPRIORITY, DICT_SHIPMODE,
  DICT_RETURNFLAG, DICT_LINESTATUS, DICT_TYPE, DICT_TPCH_MFGR, DICT_N
};

/* TPC-H nations in nationkey order, with their regionkey. */
static const char* NATION_NAMES[25] = {
  "ALGERIA", "ARGENTINA", "BRAZIL", "CANADA", "EGYPT", "ETHIOPIA", "FRANCE",
  "GERMANY", "INDIA", "INDONESIA", "IRAN", "IRAQ", "JAPAN", "JORDAN", "KENYA",
  "MOROCCO", "MOZAMBIQUE", "PERU", "CHINA", "ROMANIA", "SAUDI ARABIA", "VIETNAM",
  "RUSSIA", "UNITED KINGDOM", "UNITED STATES"};
static const int NATION_REGION[25] = {0, 1, 1, 1, 4, 0, 3, 3, 2, 2, 4, 4, 2, 4, 0,
                                      0, 0, 1, 2, 3, 4, 2, 3, 3, 1};
static const char* REGION_NAMES[5] = {"AFRICA", "AMERICA", "ASIA", "EUROPE", "MIDDLE EAST"};
static const char* SEGMENTS[5] = {"AUTOMOBILE", "BUILDING", "FURNITURE", "HOUSEHOLD", "MACHINERY"};
static const char* PRIORITIES[5] = {"1-URGENT", "2-HIGH", "3-MEDIUM", "4-NOT SPECI", "5-LOW"};
static const char* SHIPMODES[7] = {"AIR", "FOB", "MAIL", "RAIL", "REG AIR", "SHIP", "TRUCK"};
static const char* MONTHS[12] = {"Jan", "Feb", "Mar", "Apr", "May", "Jun",
                                 "Jul", "Aug", "Sep", "Oct", "Nov", "Dec"};
static const char* RETURNFLAGS[3] = {"A", "N", "R"};
static const char* LINESTATUS[2] = {"F", "O"};
/* TPC-H p_type = one syllable of each list (150 types), p_mfgr = Manufacturer#1..5 */
static const char* TYPE_S1[6] = {"STANDARD", "SMALL", "MEDIUM", "LARGE", "ECONOMY", "PROMO"};
static const char* TYPE_S2[5] = {"ANODIZED", "BURNISHED", "PLATED", "POLISHED", "BRUSHED"};
static const char* TYPE_S3[5] = {"TIN", "NICKEL", "BRASS", "STEEL", "COPPER"};
static int g_type_code[6][5][5];    /* (s1, s2, s3) -> code in DICT_TYPE */

typedef struct { int n; char** s; } dict_t;
static dict_t g_dict[DICT_N];
/* rank maps from generator-native ids to dictionary codes */
static int g_nation_code[25];       /* nationkey -> code in DICT_NATION */
static int g_city_code[25][10];     /* (nationkey, digit) -> code in DICT_CITY */
static int g_brand_code[5][5][40];  /* (m-1, c-1, b-1) -> code in DICT_BRAND1 */
static int g_ym_code[7][12];        /* (year-1992, month-1) -> code in DICT_YEARMONTH */
static int g_init_done = 0;

static int cmpstr(const void* a, const void* b) {
  return strcmp(*(char* const*)a, *(char* const*)b);
}
static void dict_build(dict_t* d, char** items, int n) {
  d->n = n; d->s = (char**)malloc(sizeof(char*) * n);
  for (int i = 0; i < n; i++) d->s[i] = items[i];
  qsort(d->s, n, sizeof(char*), cmpstr);
}
static int dict_rank(const dict_t* d, const char* s) {
  int lo = 0, hi = d->n - 1;
  while (lo <= hi) {
    int mid = (lo + hi) / 2; int c = strcmp(d->s[mid], s);
    if (c == 0) return mid;
    if (c < 0) lo = mid + 1; else hi = mid - 1;
  }
  return -1;
}
static char* xstrdup(const char* s) { char* r = (char*)malloc(strlen(s) + 1); strcpy(r, s); return r; }
static void city_name(char* out, int nation, int digit) {
  /* first 9 characters of the nation name, space padded, plus one digit */
  const char* nm = NATION_NAMES[nation]; int L = (int)strlen(nm); int k;
  for (k = 0; k < 9; k++) out[k] = k < L ? nm[k] : ' ';
  out[9] = (char)('0' + digit); out[10] = 0;
}
static void init_dicts(void) {
  if (g_init_done) return;
  char* tmp[1024]; char buf[64]; int n, i, j, k;
  for (i = 0; i < 25; i++) tmp[i] = xstrdup(NATION_NAMES[i]);
  dict_build(&g_dict[DICT_NATION], tmp, 25);
  for (i = 0; i < 5; i++) tmp[i] = xstrdup(REGION_NAMES[i]);
  dict_build(&g_dict[DICT_REGION], tmp, 5);
  n = 0;
  for (i = 0; i < 25; i++) for (j = 0; j < 10; j++) { city_name(buf, i, j); tmp[n++] = xstrdup(buf); }
  dict_build(&g_dict[DICT_CITY], tmp, n);
  for (i = 0; i < 5; i++) { sprintf(buf, "MFGR#%d", i + 1); tmp[i] = xstrdup(buf); }
  dict_build(&g_dict[DICT_MFGR], tmp, 5);
  n = 0;
  for (i = 0; i < 5; i++) for (j = 0; j < 5; j++) { sprintf(buf, "MFGR#%d%d", i + 1, j + 1); tmp[n++] = xstrdup(buf); }
  dict_build(&g_dict[DICT_CATEGORY], tmp, n);
  {
    char** big = (char**)malloc(sizeof(char*) * 1000); n = 0;
    for (i = 0; i < 5; i++) for (j = 0; j < 5; j++) for (k = 0; k < 40; k++) {
      sprintf(buf, "MFGR#%d%d%d", i + 1, j + 1, k + 1); big[n++] = xstrdup(buf);
    }
    dict_build(&g_dict[DICT_BRAND1], big, n); free(big);
  }
  n = 0;
  for (i = 0; i < 7; i++) for (j = 0; j < 12; j++) { sprintf(buf, "%s%d", MONTHS[j], 1992 + i); tmp[n++] = xstrdup(buf); }
  dict_build(&g_dict[DICT_YEARMONTH], tmp, n);
  for (i = 0; i < 5; i++) tmp[i] = xstrdup(SEGMENTS[i]);
  dict_build(&g_dict[DICT_MKTSEGMENT], tmp, 5);
  for (i = 0; i < 5; i++) tmp[i] = xstrdup(PRIORITIES[i]);
  dict_build(&g_dict[DICT_ORDERPRIORITY], tmp, 5);
  for (i = 0; i < 7; i++) tmp[i] = xstrdup(SHIPMODES[i]);
  dict_build(&g_dict[DICT_SHIPMODE], tmp, 7);
  for (i = 0; i < 3; i++) tmp[i] = xstrdup(RETURNFLAGS[i]);
  dict_build(&g_dict[DICT_RETURNFLAG], tmp, 3);
  for (i = 0; i < 2; i++) tmp[i] = xstrdup(LINESTATUS[i]);
  dict_build(&g_dict[DICT_LINESTATUS], tmp, 2);
  n = 0;
  for (i = 0; i < 6; i++) for (j = 0; j < 5; j++) for (k = 0; k < 5; k++) {
    sprintf(buf, "%s %s %s", TYPE_S1[i], TYPE_S2[j], TYPE_S3[k]); tmp[n++] = xstrdup(buf);
  }
  dict_build(&g_dict[DICT_TYPE], tmp, n);
  for (i = 0; i < 6; i++) for (j = 0; j < 5; j++) for (k = 0; k < 5; k++) {
    sprintf(buf, "%s %s %s", TYPE_S1[i], TYPE_S2[j], TYPE_S3[k]);
    g_type_code[i][j][k] = dict_rank(&g_dict[DICT_TYPE], buf);
  }
  for (i = 0; i < 5; i++) { sprintf(buf, "Manufacturer#%d", i + 1); tmp[i] = xstrdup(buf); }
  dict_build(&g_dict[DICT_TPCH_MFGR], tmp, 5);

  for (i = 0; i < 25; i++) g_nation_code[i] = dict_rank(&g_dict[DICT_NATION], NATION_NAMES[i]);
  for (i = 0; i < 25; i++) for (j = 0; j < 10; j++) {
    city_name(buf, i, j); g_city_code[i][j] = dict_rank(&g_dict[DICT_CITY], buf);
  }
  for (i = 0; i < 5; i++) for (j = 0; j < 5; j++) for (k = 0; k < 40; k++) {
    sprintf(buf, "MFGR#%d%d%d", i + 1, j + 1, k + 1);
    g_brand_code[i][j][k] = dict_rank(&g_dict[DICT_BRAND1], buf);
  }
  for (i = 0; i < 7; i++) for (j = 0; j < 12; j++) {
    sprintf(buf, "%s%d", MONTHS[j], 1992 + i); g_ym_code[i][j] = dict_rank(&g_dict[DICT_YEARMONTH], buf);
  }
  g_init_done = 1;
}
int ddqgen_dict_size(int dict) { init_dicts(); return (dict >= 0 && dict < DICT_N) ? g_dict[dict].n : -1; }
const char* ddqgen_dict_entry(int dict, int idx) {
  init_dicts();
  if (dict < 0 || dict >= DICT_N || idx < 0 || idx >= g_dict[dict].n) return NULL;
  return g_dict[dict].s[idx];
}

/* ---------------------------------------------------------------- calendar */
/* days since 1970-01-01 -> civil date (proleptic Gregorian) */
static void civil_from_days(int64_t z, int* y, int* m, int* d) {
  z += 719468;
  int64_t era = (z >= 0 ? z : z - 146096) / 146097;
  unsigned doe = (unsigned)(z - era * 146097);
  unsigned yoe = (doe - doe / 1460 + doe / 36524 - doe / 146096) / 365;
  int64_t yy = (int64_t)yoe + era * 400;
  unsigned doy = doe - (365 * yoe + yoe / 4 - yoe / 100);
  unsigned mp = (5 * doy + 2) / 153;
  unsigned dd = doy - (153 * mp + 2) / 5 + 1;
  unsigned mm = mp < 10 ? mp + 3 : mp - 9;
  *y = (int)(yy + (mm <= 2)); *m = (int)mm; *d = (int)dd;
}
static const int64_t EPOCH_1992 = 8035; /* days from 1970-01-01 to 1992-01-01 */
static int32_t datekey_of_index(int64_t idx) { /* idx days after 1992-01-01 */
  int y, m, d; civil_from_days(EPOCH_1992 + idx, &y, &m, &d); return y * 10000 + m * 100 + d;
}
static int is_leap(int y) { return (y % 4 == 0 && y % 100 != 0) || y % 400 == 0; }
static int day_of_year(int y, int m, int d) {
  static const int cum[12] = {0, 31, 59, 90, 120, 151, 181, 212, 243, 273, 304, 334};
  return cum[m - 1] + d + (m > 2 && is_leap(y));
}
int32_t ddqgen_datekey_of_index(int64_t idx) { return datekey_of_index(idx); }
/* TPC-H p_type code of syllables (s1, s2, s3) (tpchgen.c) */
int ddqgen_type_code(int s1, int s2, int s3) { init_dicts(); return g_type_code[s1][s2][s3]; }

/* ------------------------------------------------------------------- sizes */
enum { T_DATE = 1, T_CUSTOMER = 2, T_SUPPLIER = 3, T_PART = 4, T_LINEORDER = 5 };
#define N_DATE 2557      /* 1992-01-01 .. 1998-12-31 */
#define N_ORDERDATES 2406 /* 1992-01-01 .. 1998-08-02 (TPC-H order-date rule) */

static int64_t scaled(double sf, double base) {
  double v = floor(base * sf + 0.5); return v < 1 ? 1 : (int64_t)v;
}
int64_t ddqgen_ssb_rows(int table, double sf) {
  switch (table) {
    case T_DATE: return N_DATE;
    case T_CUSTOMER: return scaled(sf, 30000.0);
    case T_SUPPLIER: return scaled(sf, 2000.0);
    case T_PART:
      if (sf >= 1.0) return (int64_t)(200000.0 * floor(1.0 + log2(sf)));
      return scaled(sf, 200000.0);
    case T_LINEORDER: return scaled(sf, 6000000.0);
  }
  return -1;
}

/* column ids -------------------------------------------------------------- */
enum { D_DATEKEY = 0, D_YEAR, D_YEARMONTHNUM, D_YEARMONTH, D_DAYNUMINYEAR, D_MONTHNUMINYEAR,
       D_WEEKNUMINYEAR };
enum { C_CUSTKEY = 0, C_CITY, C_NATION, C_REGION, C_MKTSEGMENT };
enum { S_SUPPKEY = 0, S_CITY, S_NATION, S_REGION };
enum { P_PARTKEY = 0, P_MFGR, P_CATEGORY, P_BRAND1, P_RETAILPRICE };
enum { LO_ORDERKEY = 0, LO_LINENUMBER, LO_CUSTKEY, LO_PARTKEY, LO_SUPPKEY, LO_ORDERDATE,
       LO_ORDERPRIORITY, LO_SHIPPRIORITY, LO_QUANTITY, LO_EXTENDEDPRICE, LO_ORDTOTALPRICE,
       LO_DISCOUNT, LO_REVENUE, LO_SUPPLYCOST, LO_TAX, LO_COMMITDATE, LO_SHIPMODE, LO_NCOLS };

/* returns element width in bytes (4 or 8), or 0 for an unknown column */
int ddqgen_ssb_width(int table, int col) {
  switch (table) {
    case T_DATE: return (col >= 0 && col <= D_WEEKNUMINYEAR) ? 4 : 0;
    case T_CUSTOMER: return (col >= 0 && col <= C_MKTSEGMENT) ? 4 : 0;
    case T_SUPPLIER: return (col >= 0 && col <= S_REGION) ? 4 : 0;
    case T_PART: return col == P_RETAILPRICE ? 8 : (col >= 0 && col < P_RETAILPRICE) ? 4 : 0;
    case T_LINEORDER:
      if (col < 0 || col >= LO_NCOLS) return 0;
      return (col >= LO_QUANTITY && col <= LO_TAX) ? 8 : 4;
  }
  return 0;
}

/* Primary-key encoding (SURVEY 8(c).2 "the kernels must not assume dense keys").
 * key_mode 0 (default): dense keys 1..n.  key_mode 1 ("sparse"): row i of an
 * n-row table gets key 1 + ((i * 0x9E3779B1) mod 2^b), b = min(30, max(22,
 * ceil(log2 n) + 5)) -- a bijection on [0, 2^b), so keys stay unique, spread over
 * >= 16x the row count and > 2^20 values: builds take the open-addressing hash
 * table (reading O24), not the direct-mapped join index.  Foreign keys
 * map through the same function; measures (prices) keep using the dense index,
 * so every query result that does not output a key is identical in both modes. */
int64_t ddqgen_key_of(int key_mode, int64_t n, int64_t i) {
  if (key_mode == 0) return i + 1;
  int b = 0;
  while (b < 62 && (1ll << b) < n) b++;
  b += 5;
  if (b < 22) b = 22;
  if (b > 30) b = 30;
  return 1 + (int64_t)(((uint64_t)i * 0x9E3779B1ull) & ((1ull << b) - 1));
}

/* TPC-H part retail price in cents (the TPC-H formula), partkey >= 1 */
static inline int64_t retailprice(int64_t k) {
  return 90000 + ((k / 10) % 20001) + 100 * (k % 1000);
}

/* draws (random-number streams) per table; stable ids, never reuse */
enum { DR_NATION = 1, DR_CITY = 2, DR_SEGMENT = 3, DR_MFGR = 4, DR_CAT = 5, DR_BRAND = 6,
       DR_CUST = 10, DR_ODATE = 11, DR_OPRIO = 12, DR_PART = 13, DR_SUPP = 14, DR_QTY = 15,
       DR_DISC = 16, DR_TAX = 17, DR_COMMIT = 18, DR_SHIPMODE = 19 };

/* one lineorder line's (qty, disc, tax, partkey) -> used for ordtotalprice siblings */
typedef struct { int64_t qty, disc, tax, pk; } line_t;
static inline line_t lo_line(uint64_t seed, int64_t i, int64_t n_p) {
  line_t L;
  L.pk = 1 + (int64_t)(H(seed, T_LINEORDER, DR_PART, (uint64_t)i) % (uint64_t)n_p);
  L.qty = 1 + (int64_t)(H(seed, T_LINEORDER, DR_QTY, (uint64_t)i) % 50u);
  L.disc = (int64_t)(H(seed, T_LINEORDER, DR_DISC, (uint64_t)i) % 11u);
  L.tax = (int64_t)(H(seed, T_LINEORDER, DR_TAX, (uint64_t)i) % 9u);
  return L;
}

static void gen_rows(uint64_t seed, double sf, int table, int col, int64_t b, int64_t e, void* out, int km) {
  int32_t* o32 = (int32_t*)out; int64_t* o64 = (int64_t*)out; int64_t i;
  if (table == T_DATE) {
    for (i = b; i < e; i++) {
      int y, m, d; civil_from_days(EPOCH_1992 + i, &y, &m, &d);
      int32_t v = 0; int doy = day_of_year(y, m, d);
      switch (col) {
        case D_DATEKEY: v = y * 10000 + m * 100 + d; break;
        case D_YEAR: v = y; break;
        case D_YEARMONTHNUM: v = y * 100 + m; break;
        case D_YEARMONTH: v = g_ym_code[y - 1992][m - 1]; break;
        case D_DAYNUMINYEAR: v = doy; break;
        case D_MONTHNUMINYEAR: v = m; break;
        case D_WEEKNUMINYEAR: v = (doy - 1) / 7 + 1; break; /* reading O12 */
      }
      o32[i - b] = v;
    }
    return;
  }
  if (table == T_CUSTOMER || table == T_SUPPLIER) {
    const int64_t n_t = ddqgen_ssb_rows(table, sf);
    for (i = b; i < e; i++) {
      int nat = (int)(H(seed, table, DR_NATION, (uint64_t)i) % 25u);
      int32_t v = 0;
      switch (col) {
        case 0: v = (int32_t)ddqgen_key_of(km, n_t, i); break;
        case 1: v = g_city_code[nat][H(seed, table, DR_CITY, (uint64_t)i) % 10u]; break;
        case 2: v = g_nation_code[nat]; break;
        case 3: v = NATION_REGION[nat]; break; /* region dict sorted == regionkey order */
        case 4: v = (int32_t)(H(seed, table, DR_SEGMENT, (uint64_t)i) % 5u); break; /* sorted == list */
      }
      o32[i - b] = v;
    }
    return;
  }
  if (table == T_PART) {
    const int64_t n_t = ddqgen_ssb_rows(T_PART, sf);
    for (i = b; i < e; i++) {
      int m = (int)(H(seed, T_PART, DR_MFGR, (uint64_t)i) % 5u);
      int c = (int)(H(seed, T_PART, DR_CAT, (uint64_t)i) % 5u);
      int br = (int)(H(seed, T_PART, DR_BRAND, (uint64_t)i) % 40u);
      switch (col) {
        case P_PARTKEY: o32[i - b] = (int32_t)ddqgen_key_of(km, n_t, i); break;
        case P_MFGR: o32[i - b] = m; break;             /* "MFGR#1".."MFGR#5" sorted */
        case P_CATEGORY: o32[i - b] = m * 5 + c; break; /* "MFGR#11".."MFGR#55" sorted */
        case P_BRAND1: o32[i - b] = g_brand_code[m][c][br]; break;
        case P_RETAILPRICE: o64[i - b] = retailprice(i + 1); break;
      }
    }
    return;
  }
  if (table == T_LINEORDER) {
    int64_t n_c = ddqgen_ssb_rows(T_CUSTOMER, sf), n_s = ddqgen_ssb_rows(T_SUPPLIER, sf);
    int64_t n_p = ddqgen_ssb_rows(T_PART, sf);
    for (i = b; i < e; i++) {
      int64_t o = i / 4;
      switch (col) {
        case LO_ORDERKEY: o32[i - b] = (int32_t)(o + 1); break;
        case LO_LINENUMBER: o32[i - b] = (int32_t)(i % 4 + 1); break;
        case LO_CUSTKEY:
          o32[i - b] = (int32_t)ddqgen_key_of(km, n_c, (int64_t)(H(seed, T_LINEORDER, DR_CUST, (uint64_t)o) % (uint64_t)n_c));
          break;
        case LO_PARTKEY: o32[i - b] = (int32_t)ddqgen_key_of(km, n_p, lo_line(seed, i, n_p).pk - 1); break;
        case LO_SUPPKEY:
          o32[i - b] = (int32_t)ddqgen_key_of(km, n_s, (int64_t)(H(seed, T_LINEORDER, DR_SUPP, (uint64_t)i) % (uint64_t)n_s));
          break;
        case LO_ORDERDATE:
          o32[i - b] = datekey_of_index((int64_t)(H(seed, T_LINEORDER, DR_ODATE, (uint64_t)o) % N_ORDERDATES)); break;
        case LO_ORDERPRIORITY: o32[i - b] = (int32_t)(H(seed, T_LINEORDER, DR_OPRIO, (uint64_t)o) % 5u); break;
        case LO_SHIPPRIORITY: o32[i - b] = 0; break;
        case LO_QUANTITY: o64[i - b] = lo_line(seed, i, n_p).qty; break;
        case LO_EXTENDEDPRICE: { line_t L = lo_line(seed, i, n_p); o64[i - b] = L.qty * retailprice(L.pk); } break;
        case LO_ORDTOTALPRICE: {
          int64_t s = 0, j;
          for (j = o * 4; j < o * 4 + 4; j++) {
            line_t L = lo_line(seed, j, n_p); int64_t ep = L.qty * retailprice(L.pk);
            s += ep * (100 - L.disc) * (100 + L.tax) / 10000; /* floor, reading O6 */
          }
          o64[i - b] = s;
        } break;
        case LO_DISCOUNT: o64[i - b] = lo_line(seed, i, n_p).disc; break;
        case LO_REVENUE: { line_t L = lo_line(seed, i, n_p);
          o64[i - b] = L.qty * retailprice(L.pk) * (100 - L.disc) / 100; } break; /* floor, O6 */
        case LO_SUPPLYCOST: o64[i - b] = 6 * retailprice(lo_line(seed, i, n_p).pk) / 10; break;
        case LO_TAX: o64[i - b] = lo_line(seed, i, n_p).tax; break;
        case LO_COMMITDATE: {
          int64_t od = (int64_t)(H(seed, T_LINEORDER, DR_ODATE, (uint64_t)o) % N_ORDERDATES);
          o32[i - b] = datekey_of_index(od + 30 + (int64_t)(H(seed, T_LINEORDER, DR_COMMIT, (uint64_t)i) % 61u));
        } break;
        case LO_SHIPMODE: o32[i - b] = (int32_t)(H(seed, T_LINEORDER, DR_SHIPMODE, (uint64_t)i) % 7u); break;
      }
    }
  }
}

/* Generate rows [row_begin, row_end) of one SSB column into out (width per
 * ddqgen_ssb_width).  Multi-threaded over row chunks; output is independent of
 * the thread count.  Returns 0 on success, -1 on bad arguments. */
int ddqgen_ssb_column_k(uint64_t seed, double sf, int table, int col, int64_t row_begin,
                        int64_t row_end, void* out, int nthreads, int key_mode) {
  init_dicts();
  int w = ddqgen_ssb_width(table, col);
  int64_t n = ddqgen_ssb_rows(table, sf);
  if (w == 0 || row_begin < 0 || row_end > n || row_begin > row_end) return -1;
  int64_t total = row_end - row_begin;
  const int64_t chunk = 1 << 16;
  int64_t nchunks = (total + chunk - 1) / chunk, c;
  if (nthreads <= 0) nthreads = 1;
#pragma omp parallel for schedule(dynamic, 4) num_threads(nthreads)
  for (c = 0; c < nchunks; c++) {
    int64_t b = row_begin + c * chunk, e = b + chunk < row_end ? b + chunk : row_end;
    gen_rows(seed, sf, table, col, b, e, (char*)out + (b - row_begin) * w, key_mode);
  }
  return 0;
}
int ddqgen_ssb_column(uint64_t seed, double sf, int table, int col, int64_t row_begin,
                      int64_t row_end, void* out, int nthreads) {
  return ddqgen_ssb_column_k(seed, sf, table, col, row_begin, row_end, out, nthreads, 0);
}
